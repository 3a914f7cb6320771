// pagerank.cu -- PageRank pull sweeps.
//
// x'_v = (1-d)/N + d * ( sum_{u->v} x_u / D_u  +  dangling / N )
// (reading R35; D = total logical out-degree, so replica copies each divide by
// the vertex's full out-degree and mass is not double counted, Theorem E3).
//
// LB pull = merge-path over (row ends + in-edges) of the CSC: every CTA gets
// a tile of exactly IPT*256 merge items (static, precomputed once), stages
// contrib[csrc[e]] (fp32, coalesced csrc stream + L2 gathers) and the tile's
// row ends in shared memory, then each thread walks IPT items accumulating in
// fp64.  Rows completing inside the tile are finalised in place (x, delta,
// next contrib, dangling mass); rows spanning tiles accumulate into ysplit and
// are finalised by a small fixup kernel.  Replicas are mirrors (R19): they are
// not recomputed; the §2.4 merge (P@28309, mean, P@28609) sets every copy.
#include <algorithm>
#include <cmath>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "ktimer.h"

namespace gx {

struct PrState {
  double delta[3];   // L1 change of x_{t+1}, accumulated into [(t+1)%3]
  double dang[3];    // sum of x_t over dangling vertices, [t%3]
  unsigned iter;
  unsigned stop;     // 1 converged, 2 max_iters
  double last_delta;
};

struct PrArgs {
  const uint32_t* crp;
  const int32_t* csrc;
  const int64_t* trow;
  const int64_t* tedge;
  int64_t tiles;
  double* x;
  float* contrib[2];
  const uint32_t* D;
  const uint8_t* kind;   // null in exact mode
  const int32_t* gid;    // null without groups
  double* gnew;
  double* ysplit;
  const int32_t* split;
  int64_t n_split;
  double base, damp, invN;
  PrState* st;
};

template <bool SLOTS>
__device__ __forceinline__ void pr_finalize(const PrArgs& a, int64_t v, double y, double addc, float* cout,
                                            double& my_delta, double& my_dang) {
  if (SLOTS) {
    if (a.kind[v] != OWNER) return;  // holes stay 0; replicas are set by the merge
  }
  double xn = addc + a.damp * y;
  if (SLOTS && a.gid) {
    int g = a.gid[v];
    if (g >= 0) {
      a.gnew[g] = xn;
      return;
    }
  }
  double xo = a.x[v];
  a.x[v] = xn;
  my_delta += fabs(xn - xo);
  uint32_t Dv = a.D[v];
  cout[v] = Dv ? (float)(xn / (double)Dv) : 0.0f;
  if (!Dv) my_dang += xn;
}

template <int IPT, bool SLOTS>
__global__ void __launch_bounds__(256) k_pr_pull(PrArgs a) {
  constexpr int TI = IPT * 256;
  __shared__ float s_val[TI];
  __shared__ uint32_t s_end[TI + 1];
  __shared__ double s_sum[TI + 1];
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* __restrict__ cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double addc = a.base + a.damp * st->dang[t % 3] * a.invN;
  double my_delta = 0, my_dang = 0;
  const int tid = threadIdx.x;
  for (int64_t tile = blockIdx.x; tile < a.tiles; tile += gridDim.x) {
    const int64_t r0 = a.trow[tile], e0 = a.tedge[tile];
    const int nR = (int)(a.trow[tile + 1] - r0), nE = (int)(a.tedge[tile + 1] - e0);
    for (int k = tid; k < nE; k += 256) s_val[k] = __ldg(cin + __ldg(a.csrc + e0 + k));
    for (int k = tid; k < nR; k += 256) s_end[k] = (uint32_t)(a.crp[r0 + k + 1] - e0);
    for (int k = tid; k <= nR; k += 256) s_sum[k] = 0.0;
    if (tid == 0) s_end[nR] = 0x7fffffffu;
    __syncthreads();
    const int total = nR + nE;
    const int d = tid * IPT;
    if (d < total) {
      int lo = max(d - nE, 0), hi = min(d, nR);
      while (lo < hi) {
        int p = (lo + hi) >> 1;
        if ((int)s_end[p] <= d - p - 1) lo = p + 1;
        else hi = p;
      }
      int i = lo, j = d - lo;
      double acc = 0.0;
      bool first = true;
#pragma unroll
      for (int k = 0; k < IPT; k++) {
        if (d + k < total) {
          if (j < (int)s_end[i]) {
            acc += (double)s_val[j];
            j++;
          } else {
            if (first) {
              atomicAdd(&s_sum[i], acc);  // may hold carries from earlier threads
              first = false;
            } else {
              s_sum[i] = acc;             // row lies entirely in this thread
            }
            acc = 0.0;
            i++;
          }
        }
      }
      if (acc != 0.0) atomicAdd(&s_sum[i], acc);
    }
    __syncthreads();
    const bool split0 = nR > 0 && (int64_t)a.crp[r0] < e0;
    for (int k = tid; k < nR; k += 256) {
      double y = s_sum[k];
      if (k == 0 && split0) {
        atomicAdd(&a.ysplit[r0], y);
      } else {
        pr_finalize<SLOTS>(a, r0 + k, y, addc, cout, my_delta, my_dang);
      }
    }
    if (tid == 0) {
      int covered = nR ? (int)s_end[nR - 1] : 0;
      if (nE > covered) atomicAdd(&a.ysplit[r0 + nR], s_sum[nR]);
    }
    __syncthreads();
  }
  double dsum = block_sum_f64(my_delta, s_red);
  __syncthreads();
  double gsum = block_sum_f64(my_dang, s_red);
  if (tid == 0) {
    if (dsum != 0.0) atomicAdd(&st->delta[(t + 1) % 3], dsum);
    if (gsum != 0.0) atomicAdd(&st->dang[(t + 1) % 3], gsum);
  }
}

template <bool SLOTS>
__global__ void __launch_bounds__(256) k_pr_fixup(PrArgs a) {
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  float* cout = a.contrib[(t + 1) & 1];
  const double addc = a.base + a.damp * st->dang[t % 3] * a.invN;
  double my_delta = 0, my_dang = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < a.n_split; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t v = a.split[i];
    double y = a.ysplit[v];
    a.ysplit[v] = 0.0;
    pr_finalize<SLOTS>(a, v, y, addc, cout, my_delta, my_dang);
  }
  double dsum = block_sum_f64(my_delta, s_red);
  __syncthreads();
  double gsum = block_sum_f64(my_dang, s_red);
  if (threadIdx.x == 0) {
    if (dsum != 0.0) atomicAdd(&st->delta[(t + 1) % 3], dsum);
    if (gsum != 0.0) atomicAdd(&st->dang[(t + 1) % 3], gsum);
  }
}

// §2.4 confluence: every copy <- mean(owner's new value, replicas' carried
// values) (P@28609, mirror reading R19); next contrib for all copies.
__global__ void k_pr_merge(PrArgs a, const int32_t* __restrict__ gptr, const int32_t* __restrict__ gslots,
                           int64_t ngroups) {
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  float* cout = a.contrib[(t + 1) & 1];
  double my_delta = 0, my_dang = 0;
  for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < ngroups; g += (int64_t)gridDim.x * blockDim.x) {
    int b = gptr[g], e = gptr[g + 1];
    int32_t o = gslots[b];
    double s = a.gnew[g];
    for (int i = b + 1; i < e; i++) s += a.x[gslots[i]];
    double mean = s / (double)(e - b);
    my_delta += fabs(mean - a.x[o]);
    uint32_t Dv = a.D[o];
    float c = Dv ? (float)(mean / (double)Dv) : 0.0f;
    for (int i = b; i < e; i++) {
      a.x[gslots[i]] = mean;
      cout[gslots[i]] = c;
    }
    if (!Dv) my_dang += mean;
  }
  double dsum = block_sum_f64(my_delta, s_red);
  __syncthreads();
  double gsum = block_sum_f64(my_dang, s_red);
  if (threadIdx.x == 0) {
    if (dsum != 0.0) atomicAdd(&st->delta[(t + 1) % 3], dsum);
    if (gsum != 0.0) atomicAdd(&st->dang[(t + 1) % 3], gsum);
  }
}

__global__ void k_pr_advance(PrState* st, double tol, int max_iters) {
  if (st->stop) return;
  unsigned t = st->iter;
  double dl = st->delta[(t + 1) % 3];
  st->last_delta = dl;
  st->delta[(t + 2) % 3] = 0.0;
  st->dang[(t + 2) % 3] = 0.0;
  st->iter = t + 1;
  if (dl < tol) st->stop = 1;
  else if ((int)(t + 1) >= max_iters) st->stop = 2;
}

template <bool SLOTS>
__global__ void k_pr_init(PrArgs a, int64_t n_slots, double x0) {
  __shared__ double s_red[32];
  double my_dang = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n_slots; v += (int64_t)gridDim.x * blockDim.x) {
    uint8_t k = SLOTS ? a.kind[v] : (uint8_t)OWNER;
    double xv = (k == HOLE) ? 0.0 : x0;
    uint32_t Dv = a.D[v];
    a.x[v] = xv;
    a.contrib[0][v] = (k != HOLE && Dv) ? (float)(xv / (double)Dv) : 0.0f;
    a.contrib[1][v] = 0.0f;
    if (k == OWNER && !Dv) my_dang += xv;
  }
  double gsum = block_sum_f64(my_dang, s_red);
  if (threadIdx.x == 0 && gsum != 0.0) atomicAdd(&a.st->dang[0], gsum);
}

void ensure_csc(gx_graph* g);  // devgraph.cu
void run_pagerank_tpv_iter(gx_graph* g, void* args, int& launches);  // tpv.cu (pull over SELL slabs)

void run_pagerank(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  ensure_csc(g);
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  GX_CHECK_ARG(g->n > 0, "empty graph");
  int64_t ns = d.n_slots;
  r.x.alloc(c, sizeof(double) * ns);
  r.contrib[0].alloc(c, sizeof(float) * ns);
  r.contrib[1].alloc(c, sizeof(float) * ns);
  r.ysplit.alloc(c, sizeof(double) * (ns + 1));
  r.gnew.alloc(c, sizeof(double) * std::max<int64_t>(d.n_groups, 1));
  r.pst.alloc(c, sizeof(PrState));
  PrArgs a;
  a.crp = d.crp.as<uint32_t>();
  a.csrc = d.csrc.as<int32_t>();
  a.trow = d.pr_tile_row.as<int64_t>();
  a.tedge = d.pr_tile_edge.as<int64_t>();
  a.tiles = d.pr_tiles;
  a.x = r.x.as<double>();
  a.contrib[0] = r.contrib[0].as<float>();
  a.contrib[1] = r.contrib[1].as<float>();
  a.D = d.D.as<uint32_t>();
  a.kind = d.identity ? nullptr : d.kind.as<uint8_t>();
  a.gid = d.n_groups ? d.gid.as<int32_t>() : nullptr;
  a.gnew = r.gnew.as<double>();
  a.ysplit = r.ysplit.as<double>();
  a.split = d.pr_split.as<int32_t>();
  a.n_split = d.pr_n_split;
  a.damp = o.damping;
  a.base = (1.0 - o.damping) / (double)g->n;
  a.invN = 1.0 / (double)g->n;
  a.st = r.pst.as<PrState>();
  const bool slots = !d.identity;

  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(r.pst.p, 0, sizeof(PrState), s));
  CUDA_OK(cudaMemsetAsync(r.ysplit.p, 0, sizeof(double) * (ns + 1), s));
  int gi = grid_for(c, ns);
  if (slots) k_pr_init<true><<<gi, 256, 0, s>>>(a, ns, 1.0 / (double)g->n);
  else k_pr_init<false><<<gi, 256, 0, s>>>(a, ns, 1.0 / (double)g->n);
  CUDA_OK(cudaGetLastError());
  int launches = 1;

  int occ = 0;
  if (slots) CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_pull<7, true>, 256, 0));
  else CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_pull<7, false>, 256, 0));
  int grid = (int)std::max<int64_t>(1, std::min<int64_t>(d.pr_tiles, (int64_t)std::max(1, occ) * c->num_sms));
  int grid_fix = (int)std::max<int64_t>(1, std::min<int64_t>((d.pr_n_split + 255) / 256, c->num_sms * 4));
  int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_groups + 255) / 256, c->num_sms * 4));

  KTimer kt(o.profile != 0, s);
  auto one_iter = [&](int& nl) {
    kt.begin();
    if (slots) k_pr_pull<7, true><<<grid, 256, 0, s>>>(a);
    else k_pr_pull<7, false><<<grid, 256, 0, s>>>(a);
    kt.end();
    if (slots) {
      if (d.pr_n_split) k_pr_fixup<true><<<grid_fix, 256, 0, s>>>(a), nl++;
    } else {
      if (d.pr_n_split) k_pr_fixup<false><<<grid_fix, 256, 0, s>>>(a), nl++;
    }
    nl++;
    if (d.n_groups) {
      k_pr_merge<<<grid_merge, 256, 0, s>>>(a, d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), d.n_groups);
      nl++;
    }
    k_pr_advance<<<1, 1, 0, s>>>(a.st, o.tol, o.max_iters);
    nl++;
  };
  int batch = std::max(1, o.check_every);
  cudaGraphExec_t gexec = nullptr;
  int per_batch = 0;
  if (o.use_graphs && !o.profile) {
    cudaGraph_t graph;
    CUDA_OK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    for (int i = 0; i < batch; i++) one_iter(per_batch);
    CUDA_OK(cudaStreamEndCapture(s, &graph));
    CUDA_OK(cudaGraphInstantiate(&gexec, graph, 0));
    CUDA_OK(cudaGraphDestroy(graph));
  }
  PrState h;
  while (true) {
    if (gexec) {
      CUDA_OK(cudaGraphLaunch(gexec, s));
      launches += per_batch;
    } else {
      for (int i = 0; i < batch; i++) one_iter(launches);
    }
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaMemcpyAsync(&h, a.st, sizeof(PrState), cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (h.stop) break;
  }
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  if (gexec) cudaGraphExecDestroy(gexec);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = (int32_t)h.iter;
  info.converged = h.stop == 1;
  info.loop_ms = ms;
  info.last_delta = h.last_delta;
  info.edges_scanned = (int64_t)h.iter * d.m_slots;
  info.vertices_active = (int64_t)h.iter * ns;
  // bytes model: 8 B per in-edge (csrc 4 + contrib gather 4) and
  // 28 B per slot (crp 4 + x read 8 + x write 8 + contrib write 4 + D 4)
  info.bytes_model = (int64_t)h.iter * (8 * d.m_slots + 28 * ns);
  info.kernel_launches = launches;
  info.sweep_launches = kt.launches();
  info.sweep_ms = kt.total_ms();
  info.sweep_bytes = info.bytes_model;
  r.have[GX_PAGERANK] = true;
}

}  // namespace gx
