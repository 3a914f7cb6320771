// kernels_common.cuh -- warp / block primitives shared by the sweep kernels.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

namespace gx {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ unsigned int warp_max_u32(unsigned int v) {
  return __reduce_max_sync(FULL, v);
}
__device__ __forceinline__ unsigned int warp_min_u32(unsigned int v) {
  return __reduce_min_sync(FULL, v);
}

__device__ __forceinline__ uint32_t warp_incl_scan_u32(uint32_t v) {
  unsigned l = lane_id();
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t t = __shfl_up_sync(FULL, v, o);
    if (l >= (unsigned)o) v += t;
  }
  return v;
}

__device__ __forceinline__ double warp_sum_f64(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}

// Block-wide sum of a double; result valid in thread 0.  `sh` >= 32 doubles.
__device__ __forceinline__ double block_sum_f64(double v, double* sh) {
  v = warp_sum_f64(v);
  unsigned w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();
  if (lane_id() == 0) sh[w] = v;
  __syncthreads();
  double r = 0;
  if (threadIdx.x < 32) {
    r = threadIdx.x < nw ? sh[threadIdx.x] : 0.0;
    r = warp_sum_f64(r);
  }
  return r;
}

__device__ __forceinline__ unsigned long long block_sum_u64(unsigned long long v, unsigned long long* sh) {
  v = warp_sum_u64(v);
  unsigned w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();
  if (lane_id() == 0) sh[w] = v;
  __syncthreads();
  unsigned long long r = 0;
  if (threadIdx.x < 32) {
    r = threadIdx.x < nw ? sh[threadIdx.x] : 0ull;
    r = warp_sum_u64(r);
  }
  return r;
}

// host-side launch helpers (util.cu)
struct Ctx;
int grid_for(Ctx* c, int64_t work, int threads = 256);
void launch_fill_u32(Ctx* c, uint32_t* a, uint32_t v, int64_t n);
void launch_iota_i32(Ctx* c, int32_t* a, int64_t n);

}  // namespace gx
