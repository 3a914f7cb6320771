// dist.cu -- partition bounds and the exchange collectives (dist.h).
#include <algorithm>

#include "dist.h"
#include "kernels_common.cuh"

namespace gx {

void comm_allreduce(Ctx* c, const void* in, void* out, size_t count, int dtype, int op);             // comm.cpp
void comm_allgatherv(Ctx* c, void* buf, const std::vector<int64_t>& off, int dtype, size_t esize);   // comm.cpp
void comm_reduce_scatterv(Ctx* c, void* buf, const std::vector<int64_t>& off, int dtype, int op, size_t esize);
// ncclDataType / ncclRedOp values (nccl.h)
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

static size_t esize(Dt dt) { return dt == Dt::F64 ? 8 : 4; }
static int nccl_dt(Dt dt) { return dt == Dt::U32 ? NCCL_UINT32 : dt == Dt::F32 ? NCCL_FLOAT32 : NCCL_FLOAT64; }
static int nccl_op(Op op) { return op == Op::MIN ? NCCL_MIN : NCCL_SUM; }

// ---- simulated ranks: P copies on one device
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
static void sim_reduce(Ctx* c, const std::vector<void*>& bufs, int64_t n) {
  if ((int)bufs.size() > 8) GX_THROW(GX_E_UNSUPPORTED, "at most 8 simulated ranks");
  PtrArr a;
  for (size_t q = 0; q < bufs.size(); q++) a.p[q] = bufs[q];
  if (n > 0) k_reduce_copies<T, MIN><<<grid_for(c, n), 256, 0, c->stream>>>(a, (int)bufs.size(), n);
  CUDA_OK(cudaGetLastError());
}

static void sim_allreduce(Ctx* c, const std::vector<void*>& bufs, int64_t n, Dt dt, Op op) {
  const bool mn = op == Op::MIN;
  if (dt == Dt::U32) mn ? sim_reduce<uint32_t, true>(c, bufs, n) : sim_reduce<uint32_t, false>(c, bufs, n);
  else if (dt == Dt::F32) mn ? sim_reduce<float, true>(c, bufs, n) : sim_reduce<float, false>(c, bufs, n);
  else mn ? sim_reduce<double, true>(c, bufs, n) : sim_reduce<double, false>(c, bufs, n);
}

// ---- hosted exchange: stage through the context's pinned host buffer
static void* host_stage(Ctx* c, size_t bytes) {
  if (c->hstage_bytes < bytes) {
    if (c->hstage) CUDA_OK(cudaFreeHost(c->hstage));
    c->hstage = nullptr;
    c->hstage_bytes = 0;
    CUDA_OK(cudaMallocHost(&c->hstage, std::max<size_t>(bytes, 4096)));
    c->hstage_bytes = std::max<size_t>(bytes, 4096);
  }
  return c->hstage;
}

static void hosted(Ctx* c, int kind, void* dbuf, int64_t n, Dt dt, Op op, const std::vector<int64_t>* off) {
  const size_t es = esize(dt);
  void* h = host_stage(c, (size_t)n * es);
  if (n) CUDA_OK(cudaMemcpyAsync(h, dbuf, (size_t)n * es, cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  const int r = c->coll(kind, h, n, (int32_t)dt, (int32_t)op, off ? off->data() : nullptr, c->world, c->coll_user);
  if (r != 0) GX_THROW(GX_E_NCCL, "hosted exchange callback failed");
  if (kind == GX_COLL_REDUCE_SCATTERV) {   // only this rank's slice is defined
    const int64_t a = (*off)[c->rank], b = (*off)[c->rank + 1];
    if (b > a)
      CUDA_OK(cudaMemcpyAsync(static_cast<char*>(dbuf) + a * es, static_cast<char*>(h) + a * es, (size_t)(b - a) * es,
                              cudaMemcpyHostToDevice, c->stream));
  } else if (n) {
    CUDA_OK(cudaMemcpyAsync(dbuf, h, (size_t)n * es, cudaMemcpyHostToDevice, c->stream));
  }
  CUDA_OK(cudaStreamSynchronize(c->stream));   // the staging buffer is reused by the next collective
}

void Exch::allreduce(const std::vector<void*>& bufs, int64_t n, Dt dt, Op op) {
  if (P <= 1 || n <= 0) return;
  if (sim) sim_allreduce(c, bufs, n, dt, op);
  else if (c->coll) hosted(c, GX_COLL_ALLREDUCE, bufs[0], n, dt, op, nullptr);
  else comm_allreduce(c, bufs[0], bufs[0], (size_t)n, nccl_dt(dt), nccl_op(op));
}

void Exch::allgatherv(const std::vector<void*>& bufs, const std::vector<int64_t>& off, Dt dt) {
  if (P <= 1) return;
  const size_t es = esize(dt);
  if (sim) {
    for (int p = 0; p < P; p++) {
      const int64_t a = off[p], b = off[p + 1];
      if (b <= a) continue;
      for (int q = 0; q < P; q++)
        if (q != p)
          CUDA_OK(cudaMemcpyAsync(static_cast<char*>(bufs[q]) + a * es, static_cast<char*>(bufs[p]) + a * es,
                                  (size_t)(b - a) * es, cudaMemcpyDeviceToDevice, c->stream));
    }
  } else if (c->coll) {
    hosted(c, GX_COLL_ALLGATHERV, bufs[0], off[P], dt, Op::SUM, &off);
  } else {
    comm_allgatherv(c, bufs[0], off, nccl_dt(dt), es);
  }
}

void Exch::reduce_scatterv(const std::vector<void*>& bufs, const std::vector<int64_t>& off, Dt dt, Op op) {
  if (P <= 1) return;
  if (sim) sim_allreduce(c, bufs, off[P], dt, op);   // a superset: every slice reduced in every copy
  else if (c->coll) hosted(c, GX_COLL_REDUCE_SCATTERV, bufs[0], off[P], dt, op, &off);
  else comm_reduce_scatterv(c, bufs[0], off, nccl_dt(dt), nccl_op(op), esize(dt));
}

}  // namespace gx
