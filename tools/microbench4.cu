// microbench4.cu -- can the TMA engine beat the LSU/L1TEX path on random
// 4-byte gathers from an L2-resident vector (the PR pull's contrib gather)?
//  (a) LSU: ld.global.nc gathers, 8 in flight per lane (the current kernel's path)
//  (b) TMA tile::gather4: the vector viewed as a 2-D tensor of 16-byte rows;
//      every lane issues one gather4 (4 rows = 64 B) per round into a per-warp
//      shared-memory ring, completion on one mbarrier per ring stage
//  (c) cp.async.bulk 1-D: every lane issues one 16-byte bulk copy per gather
// Indices come from a precomputed stream (like the slab), values are summed.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb4 tools/microbench4.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x)                                                                   \
  do {                                                                          \
    cudaError_t e = (x);                                                        \
    if (e != cudaSuccess) {                                                     \
      printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
      return 1;                                                                 \
    }                                                                           \
  } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned par) {
  asm volatile(
      "{\n .reg .pred p;\nW_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}\n" ::"r"(
          smem_u32(b)),
      "r"(par)
      : "memory");
}

__global__ void k_lsu(const float* __restrict__ a, const uint32_t* __restrict__ idx, int64_t m, float* out) {
  float acc = 0;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < m; i += st * 8) {
    uint32_t k[8];
#pragma unroll
    for (int j = 0; j < 8; j++) k[j] = i + j * st < m ? __ldcs(idx + i + j * st) : 0u;
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) v[j] = __ldg(a + k[j]);
#pragma unroll
    for (int j = 0; j < 8; j++) acc += v[j];
  }
  if (acc == 1234.5f) out[0] = acc;
}

constexpr int STAGES = 4;
constexpr int WARPS = 8;

// (b) gather4: per round a warp gathers 128 indices (4 per lane)
__global__ void __launch_bounds__(WARPS * 32) k_tma_g4(const __grid_constant__ CUtensorMap tm, const uint32_t* __restrict__ idx,
                                                       int64_t m, float* out) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[WARPS][STAGES];
  const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float* ring = reinterpret_cast<float*>(sm) + w * STAGES * 1024;  // 32 lanes x 128 B (TMA dst alignment) per stage
  if (lane == 0)
    for (int s = 0; s < STAGES; s++) mbar_init(&bar[w][s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t rounds = m / 128;
  float acc = 0;
  uint4 keep[STAGES];
  int64_t r = gw;
  int issued = 0;
  unsigned ph[STAGES] = {0, 0, 0, 0};
  auto issue = [&](int s, int64_t rr) {
    const uint4 k = __ldcs(reinterpret_cast<const uint4*>(idx + rr * 128) + lane);
    keep[s] = k;
    if (lane == 0) mbar_expect_tx(&bar[w][s], 2048);
    __syncwarp();
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(smem_u32(ring + s * 1024 + lane * 32)),
        "l"(&tm), "r"(smem_u32(&bar[w][s])), "r"(0), "r"((int)(k.x >> 2)), "r"((int)(k.y >> 2)), "r"((int)(k.z >> 2)),
        "r"((int)(k.w >> 2))
        : "memory");
  };
  for (int s = 0; s < STAGES && r + (int64_t)s * nw < rounds; s++, issued++) issue(s, r + (int64_t)s * nw);
  int s = 0;
  while (issued > 0) {
    mbar_wait(&bar[w][s], ph[s]);
    ph[s] ^= 1;
    const uint4 k = keep[s];
    const float* b = ring + s * 1024 + lane * 32;
    acc += b[0 + (k.x & 3)] + b[4 + (k.y & 3)] + b[8 + (k.z & 3)] + b[12 + (k.w & 3)];
    __syncwarp();
    issued--;
    const int64_t nr = r + (int64_t)STAGES * nw;
    if (nr < rounds) {
      issue(s, nr);
      issued++;
    }
    r += nw;
    s = (s + 1) % STAGES;
  }
  if (acc == 1234.5f) out[0] = acc;
}

// (c) cp.async.bulk 16 B per gather (one per lane per round, 32 per round)
__global__ void __launch_bounds__(WARPS * 32) k_bulk16(const float* __restrict__ a, const uint32_t* __restrict__ idx,
                                                       int64_t m, float* out) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[WARPS][STAGES];
  const unsigned lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float* ring = reinterpret_cast<float*>(sm) + w * STAGES * 128;   // 32 lanes x 16 B per stage
  if (lane == 0)
    for (int s = 0; s < STAGES; s++) mbar_init(&bar[w][s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t rounds = m / 32;
  float acc = 0;
  uint32_t keep[STAGES];
  unsigned ph[STAGES] = {0, 0, 0, 0};
  int64_t r = gw;
  int issued = 0;
  auto issue = [&](int s, int64_t rr) {
    const uint32_t k = __ldcs(idx + rr * 32 + lane);
    keep[s] = k;
    if (lane == 0) mbar_expect_tx(&bar[w][s], 512);
    __syncwarp();
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16, [%2];" ::"r"(
            smem_u32(ring + s * 128 + lane * 4)),
        "l"(a + (k & ~3u)), "r"(smem_u32(&bar[w][s]))
        : "memory");
  };
  for (int s = 0; s < STAGES && r + (int64_t)s * nw < rounds; s++, issued++) issue(s, r + (int64_t)s * nw);
  int s = 0;
  while (issued > 0) {
    mbar_wait(&bar[w][s], ph[s]);
    ph[s] ^= 1;
    acc += ring[s * 128 + lane * 4 + (keep[s] & 3)];
    __syncwarp();
    issued--;
    const int64_t nr = r + (int64_t)STAGES * nw;
    if (nr < rounds) {
      issue(s, nr);
      issued++;
    }
    r += nw;
    s = (s + 1) % STAGES;
  }
  if (acc == 1234.5f) out[0] = acc;
}

__global__ void k_fill_idx(uint32_t* idx, int64_t m, uint32_t mask) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t x = (uint64_t)i * 0x9E3779B97F4A7C15ull;
    x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33;
    idx[i] = (uint32_t)x & mask;
  }
}

int main() {
  const int64_t n = 16 << 20;   // 64 MB of floats (RMAT-24 contrib)
  const int64_t m = 256 << 20;  // 256M gathers (~ one RMAT-24 sweep)
  float *a, *out;
  uint32_t* idx;
  CK(cudaMalloc(&a, n * 4));
  CK(cudaMalloc(&idx, m * 4));
  CK(cudaMalloc(&out, 4));
  CK(cudaMemset(a, 0, n * 4));
  k_fill_idx<<<1184, 256>>>(idx, m, (uint32_t)(n - 1));
  CK(cudaDeviceSynchronize());
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));

  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  CUtensorMap tm;
  cuuint64_t gdim[2] = {4, (cuuint64_t)(n / 4)};
  cuuint64_t gstr[1] = {16};
  cuuint32_t box[2] = {4, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult cr = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, a, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) printf("tensor map encode failed: %d\n", (int)cr);

  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto timeit = [&](const char* name, auto launch) {
    launch();
    cudaDeviceSynchronize();
    float best = 1e9;
    for (int i = 0; i < 5; i++) {
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      best = ms < best ? ms : best;
    }
    cudaError_t err = cudaGetLastError();
    printf("%-28s %8.3f ms  %7.1f Ggather/s  %s\n", name, best, m / (best * 1e-3) / 1e9,
           err == cudaSuccess ? "" : cudaGetErrorString(err));
  };
  for (int occ : {4, 8}) {
    char nm[64];
    snprintf(nm, sizeof nm, "LSU ldg.nc x8 (occ %d)", occ);
    timeit(nm, [&] { k_lsu<<<sms * occ, 256>>>(a, idx, m, out); });
  }
  const int smem_g4 = WARPS * STAGES * 4096, smem_b = WARPS * STAGES * 512;
  for (int occ : {2, 4, 8}) {
    char nm[64];
    snprintf(nm, sizeof nm, "bulk 16B (CTA/SM %d)", occ);
    timeit(nm, [&] { k_bulk16<<<sms * occ, WARPS * 32, smem_b>>>(a, idx, m, out); });
  }
  cudaFuncSetAttribute(k_tma_g4, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_g4);
  for (int occ : {1}) {
    char nm[64];
    snprintf(nm, sizeof nm, "TMA gather4 (CTA/SM %d)", occ);
    timeit(nm, [&] { k_tma_g4<<<sms * occ, WARPS * 32, smem_g4>>>(tm, idx, m, out); });
  }
  return 0;
}
