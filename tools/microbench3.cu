// microbench3.cu -- what limits random 4-byte gathers on B200?
//  (a) array size sweep incl. L1-resident sizes, L1-allocating vs L2-only loads
//  (b) lines per warp instruction: 32 lanes spread over k distinct 128 B lines
//  (c) shared-memory random gathers, (d) distributed shared memory in a cluster
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb3 tools/microbench3.cu
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__device__ __forceinline__ uint32_t hsh(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return (uint32_t)x;
}

template <int MODE>   // 0 ld.global.ca (L1 allocate), 1 ld.global.cg (L2 only), 2 ld.global.nc
__global__ void gather(const float* __restrict__ a, uint32_t mask, int64_t n, float* out) {
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st * 8) {
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) {
      uint32_t k = hsh(i + j * st) & mask;
      if (MODE == 0) v[j] = __ldca(a + k);
      else if (MODE == 1) v[j] = __ldcg(a + k);
      else v[j] = __ldg(a + k);
    }
#pragma unroll
    for (int j = 0; j < 8; j++) acc += v[j];
  }
  if (acc == 1234.5f) out[0] = acc;
}

// lanes grouped: 32/k lanes share one random line (distinct words inside it)
__global__ void gather_lines(const float* __restrict__ a, uint32_t line_mask, int k, int64_t n, float* out) {
  float acc = 0;
  const unsigned lane = threadIdx.x & 31, grp = lane / (32 / k), sub = lane % (32 / k);
  int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = wid; i * 32 < n; i += nw * 8) {
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) {
      uint32_t line = hsh((i + j * nw) * 64 + grp) & line_mask;
      v[j] = __ldcg(a + line * 32 + (sub % 32));
    }
#pragma unroll
    for (int j = 0; j < 8; j++) acc += v[j];
  }
  if (acc == 1234.5f) out[0] = acc;
}

__global__ void smem_gather(int64_t n, float* out, uint32_t mask) {
  extern __shared__ float s[];
  for (uint32_t i = threadIdx.x; i <= mask; i += blockDim.x) s[i] = (float)i;
  __syncthreads();
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st * 8) {
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) v[j] = s[hsh(i + j * st) & mask];
#pragma unroll
    for (int j = 0; j < 8; j++) acc += v[j];
  }
  if (acc == 1234.5f) out[0] = acc;
}

__global__ void dsmem_gather(int64_t n, float* out, uint32_t mask) {
  extern __shared__ float s[];
  cg::cluster_group cl = cg::this_cluster();
  for (uint32_t i = threadIdx.x; i <= mask; i += blockDim.x) s[i] = (float)i;
  cl.sync();
  const unsigned nb = cl.num_blocks();
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st * 8) {
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) {
      uint32_t h = hsh(i + j * st);
      const float* r = cl.map_shared_rank(s, (h >> 24) % nb);
      v[j] = r[h & mask];
    }
#pragma unroll
    for (int j = 0; j < 8; j++) acc += v[j];
  }
  cl.sync();
  if (acc == 1234.5f) out[0] = acc;
}

template <class F>
float timeit(F f) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < 4; r++) {
    cudaEventRecord(e0); f(); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (r && ms < best) best = ms;
  }
  return best;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t n = 1ll << 28;
  float* a; cudaMalloc(&a, 1ull << 28); cudaMemset(a, 0, 1ull << 28);
  float* out; cudaMalloc(&out, 64);
  const int grid = sms * 8;
  for (int lg = 13; lg <= 26; lg += (lg < 18 ? 1 : 2)) {
    uint32_t mask = (1u << lg) - 1;
    float t0 = timeit([&] { gather<0><<<grid, 256>>>(a, mask, n, out); });
    float t1 = timeit([&] { gather<1><<<grid, 256>>>(a, mask, n, out); });
    float t2 = timeit([&] { gather<2><<<grid, 256>>>(a, mask, n, out); });
    printf("array %8.3f MB: ca %6.1f  cg %6.1f  nc %6.1f Ggather/s\n", (4.0 * (mask + 1)) / (1 << 20), n / t0 / 1e6,
           n / t1 / 1e6, n / t2 / 1e6);
  }
  for (int k = 1; k <= 32; k *= 2) {
    float t = timeit([&] { gather_lines<<<grid, 256>>>(a, (1u << 19) - 1, k, n, out); });
    printf("lines/instr %2d (64 MB array, cg): %6.1f Ggather/s  %6.1f Glines/s\n", k, n / t / 1e6, n / t / 1e6 * k / 32);
  }
  cudaFuncSetAttribute(smem_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 << 10);
  for (int lg = 10; lg <= 15; lg++) {
    uint32_t mask = (1u << lg) - 1;
    float t = timeit([&] { smem_gather<<<sms, 1024, (mask + 1) * 4>>>(n, out, mask); });
    printf("smem %6.1f KB: %7.1f Ggather/s\n", 4.0 * (mask + 1) / 1024, n / t / 1e6);
  }
  cudaFuncSetAttribute(dsmem_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 << 10);
  cudaFuncSetAttribute(dsmem_gather, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int cs = 1; cs <= 16; cs *= 2) {
    uint32_t mask = (1u << 15) - 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(sms / cs * cs); cfg.blockDim = dim3(1024); cfg.dynamicSmemBytes = (mask + 1) * 4;
    cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = cs;
    at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1; cfg.attrs = at; cfg.numAttrs = 1;
    float t = timeit([&] { cudaLaunchKernelEx(&cfg, dsmem_gather, n, out, mask); });
    cudaError_t e = cudaGetLastError();
    printf("dsmem cluster %2d (128 KB/CTA): %7.1f Ggather/s %s\n", cs, n / t / 1e6, e ? cudaGetErrorString(e) : "");
  }
  return 0;
}
