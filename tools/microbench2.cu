// microbench2.cu -- does an L2 eviction-priority hint keep a 64 MB gathered
// vector resident while a 1 GB stream flows through L2?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return (uint32_t)x;
}
__device__ __forceinline__ uint64_t pol_first() { uint64_t p; asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ uint64_t pol_last() { uint64_t p; asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p)); return p; }
__device__ __forceinline__ uint64_t pol_normal() { uint64_t p; asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p)); return p; }

template <int SP, int GP>   // 0 plain, 1 evict_first, 2 evict_last, 3 evict_normal
__global__ void mix(const uint4* __restrict__ big, int64_t nbig, const float* __restrict__ a, uint32_t mask, float* out) {
  uint64_t ps = SP == 1 ? pol_first() : SP == 2 ? pol_last() : pol_normal();
  uint64_t pg = GP == 1 ? pol_first() : GP == 2 ? pol_last() : pol_normal();
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < nbig; i += st) {
    uint4 r;
    if (SP == 0) r = __ldg(big + i);
    else asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(big + i), "l"(ps));
    uint32_t k[4] = {hsh(r.x + i) & mask, hsh(r.y + 2 * i) & mask, hsh(r.z + 3 * i) & mask, hsh(r.w + 4 * i) & mask};
#pragma unroll
    for (int j = 0; j < 4; j++) {
      float v;
      if (GP == 0) v = __ldg(a + k[j]);
      else asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(a + k[j]), "l"(pg));
      acc += v;
    }
  }
  if (acc == 1234.5f) out[0] = acc;
}

// stream only (bandwidth reference)
__global__ void stream_only(const uint4* __restrict__ big, int64_t nbig, float* out) {
  uint32_t acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < nbig; i += st) { uint4 r = __ldg(big + i); acc ^= r.x ^ r.w; }
  if (acc == 12345u) out[0] = acc;
}

template <int SP, int GP>
float run(const uint4* big, int64_t nbig, const float* a, uint32_t mask, float* out, int sms) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms = 0;
  for (int r = 0; r < 3; r++) {
    cudaEventRecord(e0); mix<SP, GP><<<sms * 8, 256>>>(big, nbig, a, mask, out); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
  }
  return ms;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  printf("L2 %d MB, persistingL2CacheMaxSize %d MB, accessPolicyMaxWindowSize %d MB\n", p.l2CacheSize >> 20,
         p.persistingL2CacheMaxSize >> 20, p.accessPolicyMaxWindowSize >> 20);
  int64_t nbig = (1ll << 30) / 16;   // 1 GB stream, 67M x 16B  -> 268M gathers
  uint4* big; cudaMalloc(&big, nbig * 16); cudaMemset(big, 1, nbig * 16);
  float* a; cudaMalloc(&a, 64 << 20); cudaMemset(a, 0, 64 << 20);
  float* out; cudaMalloc(&out, 4);
  uint32_t mask = (16u << 20) - 1;
  {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms = 0;
    for (int r = 0; r < 3; r++) { cudaEventRecord(e0); stream_only<<<sms * 8, 256>>>(big, nbig, out); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); }
    printf("stream only 1 GB: %.3f ms  %.0f GB/s\n", ms, 1024.0 / ms);
  }
  for (int pers = 0; pers < 2; pers++) {
    if (pers) {
      size_t want = p.persistingL2CacheMaxSize;
      cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want);
      size_t got = 0; cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize);
      printf("set persisting limit -> %s, now %zu MB\n", cudaGetErrorString(e), got >> 20);
    }
    float t;
    t = run<0, 0>(big, nbig, a, mask, out, sms); printf("pers=%d stream plain  / gather plain : %.3f ms  %.1f Ggather/s\n", pers, t, 4.0 * nbig / t / 1e6);
    t = run<1, 0>(big, nbig, a, mask, out, sms); printf("pers=%d stream first  / gather plain : %.3f ms  %.1f Ggather/s\n", pers, t, 4.0 * nbig / t / 1e6);
    t = run<1, 2>(big, nbig, a, mask, out, sms); printf("pers=%d stream first  / gather last  : %.3f ms  %.1f Ggather/s\n", pers, t, 4.0 * nbig / t / 1e6);
    t = run<1, 3>(big, nbig, a, mask, out, sms); printf("pers=%d stream first  / gather normal: %.3f ms  %.1f Ggather/s\n", pers, t, 4.0 * nbig / t / 1e6);
    t = run<3, 2>(big, nbig, a, mask, out, sms); printf("pers=%d stream normal / gather last  : %.3f ms  %.1f Ggather/s\n", pers, t, 4.0 * nbig / t / 1e6);
  }
  return 0;
}
