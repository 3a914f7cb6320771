// dist.cu -- partition bounds and the exchange collectives (dist.h).
#include <algorithm>

#include "dist.h"
#include "kernels_common.cuh"

namespace gx {

void comm_allreduce(Ctx* c, const void* in, void* out, size_t count, int dtype, int op);  // comm.cpp
enum { NCCL_UINT32 = 3, NCCL_FLOAT32 = 7, NCCL_FLOAT64 = 8 };
enum { NCCL_SUM = 0, NCCL_MIN = 3 };

std::vector<int64_t> partition_rows(const std::vector<int64_t>& rp, int64_t n, int P, int64_t align) {
  std::vector<int64_t> b(P + 1, 0);
  const int64_t m = rp[n];
  for (int p = 1; p < P; p++) {
    // first row whose prefix (edges + rows, so empty rows still count) reaches p/P of the total
    const long double target = (long double)(m + n) * p / P;
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t mid = (lo + hi) / 2;
      if ((long double)(rp[mid] + mid) < target) lo = mid + 1;
      else hi = mid;
    }
    int64_t r = (lo + align / 2) / align * align;
    r = std::max(b[p - 1], std::min(r, n));
    b[p] = r;
  }
  b[P] = n;
  return b;
}

std::vector<int64_t> partition_rows_dev(Ctx* c, const uint32_t* rp_dev, int64_t n, int P, int64_t align) {
  std::vector<uint32_t> h(n + 1);
  CUDA_OK(cudaMemcpyAsync(h.data(), rp_dev, sizeof(uint32_t) * (n + 1), cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  std::vector<int64_t> rp(h.begin(), h.end());
  return partition_rows(rp, n, P, align);
}

struct PtrArr {
  void* p[8];
};

template <class T, bool MIN>
__global__ void k_reduce_copies(PtrArr a, int P, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    T v = reinterpret_cast<T*>(a.p[0])[i];
    for (int q = 1; q < P; q++) {
      const T x = reinterpret_cast<T*>(a.p[q])[i];
      v = MIN ? (x < v ? x : v) : v + x;
    }
    for (int q = 0; q < P; q++) reinterpret_cast<T*>(a.p[q])[i] = v;
  }
}

template <class T, bool MIN>
static void sim_reduce(Ctx* c, const std::vector<T*>& bufs, int64_t n) {
  if ((int)bufs.size() > 8) GX_THROW(GX_E_UNSUPPORTED, "at most 8 simulated ranks");
  PtrArr a;
  for (size_t q = 0; q < bufs.size(); q++) a.p[q] = bufs[q];
  if (n > 0) k_reduce_copies<T, MIN><<<grid_for(c, n), 256, 0, c->stream>>>(a, (int)bufs.size(), n);
  CUDA_OK(cudaGetLastError());
}

void Exch::min_u32(const std::vector<uint32_t*>& bufs, int64_t n) {
  if (sim) sim_reduce<uint32_t, true>(c, bufs, n);
  else if (P > 1) comm_allreduce(c, bufs[0], bufs[0], (size_t)n, NCCL_UINT32, NCCL_MIN);
}
void Exch::sum_f32(const std::vector<float*>& bufs, int64_t n) {
  if (sim) sim_reduce<float, false>(c, bufs, n);
  else if (P > 1) comm_allreduce(c, bufs[0], bufs[0], (size_t)n, NCCL_FLOAT32, NCCL_SUM);
}
void Exch::sum_f64(const std::vector<double*>& bufs, int64_t n) {
  if (sim) sim_reduce<double, false>(c, bufs, n);
  else if (P > 1) comm_allreduce(c, bufs[0], bufs[0], (size_t)n, NCCL_FLOAT64, NCCL_SUM);
}
void Exch::sum_u32(const std::vector<uint32_t*>& bufs, int64_t n) {
  if (sim) sim_reduce<uint32_t, false>(c, bufs, n);
  else if (P > 1) comm_allreduce(c, bufs[0], bufs[0], (size_t)n, NCCL_UINT32, NCCL_SUM);
}

}  // namespace gx
