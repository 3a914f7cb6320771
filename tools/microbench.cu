// microbench.cu -- calibrate random 4-byte gather / atomicMin throughput on
// B200 (the ceiling of the PR pull and SSSP relax kernels).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return (uint32_t)x;
}

template <int U>
__global__ void gather_hash(const float* __restrict__ a, uint32_t mask, int64_t n, float* out) {
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid * U; i < n; i += st * U) {
    float v[U];
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = __ldg(a + (hsh(i + u) & mask));
#pragma unroll
    for (int u = 0; u < U; u++) acc += v[u];
  }
  if (acc == 12345.f) out[0] = acc;
}

// index stream + gather (the PR pattern): idx read coalesced
template <int U>
__global__ void gather_idx(const float* __restrict__ a, const uint32_t* __restrict__ idx, int64_t n, float* out) {
  float acc = 0;
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st * U) {
    uint32_t k[U];
#pragma unroll
    for (int u = 0; u < U; u++) k[u] = (i + u * st < n) ? __ldg(idx + i + u * st) : 0;
#pragma unroll
    for (int u = 0; u < U; u++) acc += __ldg(a + k[u]);
  }
  if (acc == 12345.f) out[0] = acc;
}

__global__ void atom_min(uint32_t* __restrict__ a, uint32_t mask, int64_t n) {
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st) atomicMin(a + (hsh(i) & mask), (uint32_t)i);
}

__global__ void fill_idx(uint32_t* idx, uint32_t mask, int64_t n) {
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n; i += st) idx[i] = hsh(i * 7 + 3) & mask;
}

int main() {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t N = 1ll << 28;  // 268M accesses
  float* out; cudaMalloc(&out, 4);
  uint32_t* idx; cudaMalloc(&idx, N * 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int lg = 22; lg <= 28; lg += 2) {   // array of 2^lg floats: 16 MB .. 1 GB
    int64_t sz = 1ll << lg;
    float* a; cudaMalloc(&a, sz * 4); cudaMemset(a, 0, sz * 4);
    uint32_t mask = (uint32_t)(sz - 1);
    float ms;
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0); gather_hash<8><<<sms * 8, 256>>>(a, mask, N, out); cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    cudaEventElapsedTime(&ms, e0, e1);
    printf("gather_hash U8  array %5lld MB: %7.1f G/s\n", (long long)(sz * 4 >> 20), N / ms / 1e6);
    fill_idx<<<sms * 8, 256>>>(idx, mask, N);
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0); gather_idx<4><<<sms * 8, 256>>>(a, idx, N, out); cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    cudaEventElapsedTime(&ms, e0, e1);
    printf("gather_idx  U4  array %5lld MB: %7.1f G/s (idx stream %.0f GB/s)\n", (long long)(sz * 4 >> 20), N / ms / 1e6, N * 4 / ms / 1e6);
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0); atom_min<<<sms * 8, 256>>>((uint32_t*)a, mask, N); cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    cudaEventElapsedTime(&ms, e0, e1);
    printf("atomicMin       array %5lld MB: %7.1f G/s\n", (long long)(sz * 4 >> 20), N / ms / 1e6);
    cudaFree(a);
  }
  for (int U : {1, 2, 4, 8}) {
    int64_t sz = 1ll << 24; float* a; cudaMalloc(&a, sz * 4); cudaMemset(a, 0, sz * 4);
    float ms = 0;
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0);
      if (U == 1) gather_hash<1><<<sms * 8, 256>>>(a, sz - 1, N, out);
      if (U == 2) gather_hash<2><<<sms * 8, 256>>>(a, sz - 1, N, out);
      if (U == 4) gather_hash<4><<<sms * 8, 256>>>(a, sz - 1, N, out);
      if (U == 8) gather_hash<8><<<sms * 8, 256>>>(a, sz - 1, N, out);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    cudaEventElapsedTime(&ms, e0, e1);
    printf("gather_hash U%d 64MB: %7.1f G/s\n", U, N / ms / 1e6);
    cudaFree(a);
  }
  return 0;
}
