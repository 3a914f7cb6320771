// util.cu -- small launch helpers and result download (owner-slot gather).
#include <algorithm>

#include "gx_internal.h"
#include "kernels_common.cuh"

namespace gx {

int grid_for(Ctx* c, int64_t work, int threads) {
  int64_t b = (work + threads - 1) / threads;
  int64_t cap = (int64_t)c->num_sms * 16;
  return (int)std::max<int64_t>(1, std::min(b, cap));
}

__global__ void k_fill_u32(uint32_t* __restrict__ a, uint32_t v, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = v;
}

__global__ void k_iota_i32(int32_t* __restrict__ a, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = (int32_t)i;
}

template <class T>
__global__ void k_gather(const T* __restrict__ src, const int32_t* __restrict__ idx, T* __restrict__ out,
                         int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = src[idx[i]];
}

void launch_fill_u32(Ctx* c, uint32_t* a, uint32_t v, int64_t n) {
  if (n <= 0) return;
  k_fill_u32<<<grid_for(c, n), 256, 0, c->stream>>>(a, v, n);
  CUDA_OK(cudaGetLastError());
}

void launch_iota_i32(Ctx* c, int32_t* a, int64_t n) {
  if (n <= 0) return;
  k_iota_i32<<<grid_for(c, n), 256, 0, c->stream>>>(a, n);
  CUDA_OK(cudaGetLastError());
}

// Results are read from owner slots (SURVEY.md §8(b) ownership; holes and
// replicas are never exposed), indexed by original vertex id.
template <class T>
static void gather_out(gx_graph* g, const DBuf& src, void* out, int64_t n, uint32_t flags, int kind) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  bool dev = flags & GX_PTRS_DEVICE;
  const T* sp = src.as<T>();
  join_download(g, kind);   // a previous asynchronous download of this kind
  if (g->dg.identity && !dev && (flags & GX_DL_ASYNC)) {
    // the copy on the second stream after the producing work; the ctx stream
    // goes on (join_download / gx_sync / destroy complete it)
    if (!c->copy_stream) CUDA_OK(cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    cudaEvent_t ev;
    CUDA_OK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    CUDA_OK(cudaEventRecord(ev, s));
    CUDA_OK(cudaStreamWaitEvent(c->copy_stream, ev, 0));
    CUDA_OK(cudaEventDestroy(ev));
    CUDA_OK(cudaMemcpyAsync(out, sp, sizeof(T) * n, cudaMemcpyDeviceToHost, c->copy_stream));
    CUDA_OK(cudaEventCreateWithFlags(&g->dl_ev[kind], cudaEventDisableTiming));
    CUDA_OK(cudaEventRecord(g->dl_ev[kind], c->copy_stream));
    return;
  }
  if (g->dg.identity) {
    CUDA_OK(cudaMemcpyAsync(out, sp, sizeof(T) * n, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s));
  } else {
    DBuf tmp;
    T* dst = (T*)out;
    if (!dev) {
      tmp.alloc(c, sizeof(T) * std::max<int64_t>(n, 1));
      dst = tmp.as<T>();
    }
    if (n) k_gather<T><<<grid_for(c, n), 256, 0, s>>>(sp, g->dg.owner.as<int32_t>(), dst, n);
    CUDA_OK(cudaGetLastError());
    if (!dev) CUDA_OK(cudaMemcpyAsync(out, dst, sizeof(T) * n, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
  }
  CUDA_OK(cudaStreamSynchronize(s));
}

// the ctx stream waits for the asynchronous download(s) of `kind` (-1: all)
// before it may overwrite or free their source buffers
void join_download(gx_graph* g, int kind) {
  for (int k = 0; k < 8; k++) {
    if ((kind >= 0 && k != kind) || !g->dl_ev[k]) continue;
    CUDA_OK(cudaStreamWaitEvent(g->ctx->stream, g->dl_ev[k], 0));
    CUDA_OK(cudaEventDestroy(g->dl_ev[k]));
    g->dl_ev[k] = nullptr;
  }
}

void download(gx_graph* g, int kind, void* out, int64_t count, uint32_t flags) {
  RunState& r = g->rs;
  switch (kind) {
    case GX_OUT_DIST_U32:
      if (!r.have[GX_SSSP]) GX_THROW(GX_E_STATE, "SSSP has not run on this graph");
      GX_CHECK_ARG(count == g->n, "count must be n");
      gather_out<uint32_t>(g, r.dist, out, count, flags, kind);
      break;
    case GX_OUT_RANK_F64:
      if (!r.have[GX_PAGERANK]) GX_THROW(GX_E_STATE, "PageRank has not run on this graph");
      GX_CHECK_ARG(count == g->n, "count must be n");
      gather_out<double>(g, r.x, out, count, flags, kind);
      break;
    case GX_OUT_LABEL_I32:
      if (!r.have[GX_SCC]) GX_THROW(GX_E_STATE, "SCC has not run on this graph");
      GX_CHECK_ARG(count == g->n, "count must be n");
      // labels are stored per original vertex already
      CUDA_OK(cudaMemcpyAsync(out, r.label2.p, sizeof(int32_t) * count,
                              (flags & GX_PTRS_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                              g->ctx->stream));
      CUDA_OK(cudaStreamSynchronize(g->ctx->stream));
      break;
    case GX_OUT_BC_F64:
      if (!r.have[GX_BC]) GX_THROW(GX_E_STATE, "BC has not run on this graph");
      GX_CHECK_ARG(count == g->n, "count must be n");
      // BC runs on G_L over original ids (algos.cu): no owner gather
      CUDA_OK(cudaMemcpyAsync(out, r.bc.p, sizeof(double) * count,
                              (flags & GX_PTRS_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                              g->ctx->stream));
      CUDA_OK(cudaStreamSynchronize(g->ctx->stream));
      break;
    case GX_OUT_MST_WEIGHT_U64:
      if (!r.have[GX_MST]) GX_THROW(GX_E_STATE, "MST has not run on this graph");
      GX_CHECK_ARG(count == 1, "count must be 1");
      if (flags & GX_PTRS_DEVICE) {
        CUDA_OK(cudaMemcpyAsync(out, &r.mst_weight, 8, cudaMemcpyHostToDevice, g->ctx->stream));
        CUDA_OK(cudaStreamSynchronize(g->ctx->stream));
      } else {
        *(uint64_t*)out = r.mst_weight;
      }
      break;
    default:
      GX_THROW(GX_E_INVALID, "unknown download kind");
  }
}

}  // namespace gx
