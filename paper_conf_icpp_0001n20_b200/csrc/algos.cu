// algos.cu -- the paper's other algorithms (PAPER.md P@36969: SSSP, MST, SCC,
// PR, BC) on the logical graph G_L: every slot edge
// with its source folded into the owner vertex (replica rows are part of the
// owner's adjacency, reading R19 "owner broadcast"), including every edge the
// transforms added.  Results are per original vertex.
//
//  * SCC: colouring (max-id forward propagation, backward closure from the
//    colour roots), repeated on the unassigned vertices; label = min original
//    id of the component (R38).  Bit-exact.
//  * MST: Boruvka on the undirected view ({u,v} weighs the lighter direction,
//    R39) with 64-bit (weight, edge) keys; minimum spanning forest weight.
//  * BC: Brandes (Alg 1, Eq 1-2, P@12652-14843), unweighted, directed, over
//    the caller's source sample (R37): level-synchronous forward pass with
//    fp64 sigma (atomicAdd, P@14089), backward delta pass per level.
#include <algorithm>
#include <chrono>
#include <cub/cub.cuh>

#include "dist.h"
#include "gx_internal.h"
#include "kernels_common.cuh"

namespace gx {

// ---------------------------------------------------------------- G_L
__global__ void k_esrc(const uint32_t* __restrict__ rp, int64_t n, uint32_t* __restrict__ esrc) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw)
    for (uint32_t e = rp[u] + lane_id(); e < rp[u + 1]; e += 32) esrc[e] = (uint32_t)u;
}

void ensure_logical(gx_graph* g) {
  DevGraph& d = g->dg;
  if (d.lg_ready) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  const int64_t n = g->n;
  if (!d.identity) {
    const SlotGraph& sg = g->sg;
    std::vector<uint32_t> rp(n + 1, 0);
    for (int64_t sl = 0; sl < sg.n_slots; sl++)
      if (sg.kind[sl] != HOLE) rp[sg.slot_to_orig[sl] + 1] += (uint32_t)(sg.rp[sl + 1] - sg.rp[sl]);
    for (int64_t u = 0; u < n; u++) rp[u + 1] += rp[u];
    std::vector<uint2> adj(std::max<uint32_t>(rp[n], 1));
    std::vector<uint32_t> cur(rp.begin(), rp.end() - 1);
    for (int64_t sl = 0; sl < sg.n_slots; sl++) {
      if (sg.kind[sl] == HOLE) continue;
      const int32_t u = sg.slot_to_orig[sl];
      for (int64_t e = sg.rp[sl]; e < sg.rp[sl + 1]; e++)
        adj[cur[u]++] = make_uint2((uint32_t)sg.slot_to_orig[sg.col[e]], sg.w[e]);
    }
    d.lg_m = rp[n];
    d.lg_rp.alloc(c, sizeof(uint32_t) * (n + 1));
    d.lg_adj.alloc(c, sizeof(uint2) * adj.size());
    CUDA_OK(cudaMemcpyAsync(d.lg_rp.p, rp.data(), sizeof(uint32_t) * (n + 1), cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(d.lg_adj.p, adj.data(), sizeof(uint2) * adj.size(), cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaStreamSynchronize(s));
  } else {
    d.lg_m = d.m_slots;
  }
  const uint32_t* rp = d.identity ? d.rp.as<uint32_t>() : d.lg_rp.as<uint32_t>();
  d.lg_esrc.alloc(c, sizeof(uint32_t) * std::max<int64_t>(d.lg_m, 1));
  if (n) k_esrc<<<grid_for(c, n * 32), 256, 0, s>>>(rp, n, d.lg_esrc.as<uint32_t>());
  CUDA_OK(cudaGetLastError());
  d.lg_ready = true;
}

struct LG {
  const uint32_t* rp;
  const uint2* adj;
  const uint32_t* esrc;
  int64_t n, m;
};

static LG logical(gx_graph* g) {
  ensure_logical(g);
  DevGraph& d = g->dg;
  LG L;
  L.rp = d.identity ? d.rp.as<uint32_t>() : d.lg_rp.as<uint32_t>();
  L.adj = d.identity ? d.adj.as<uint2>() : d.lg_adj.as<uint2>();
  L.esrc = d.lg_esrc.as<uint32_t>();
  L.n = g->n;
  L.m = d.lg_m;
  return L;
}

#define GRID_STRIDE(i, n) for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

// ---------------------------------------------------------------- SCC
__global__ void k_scc_color_init(const int32_t* __restrict__ label, uint32_t* __restrict__ color,
                                 uint8_t* __restrict__ vis, int64_t n) {
  GRID_STRIDE(v, n) {
    if (label[v] < 0) color[v] = (uint32_t)v;
    vis[v] = 0;
  }
}
// forward max-colour propagation over the edges of unassigned vertices
__global__ void k_scc_fw(LG L, const int32_t* __restrict__ label, uint32_t* __restrict__ color, int* __restrict__ changed) {
  int ch = 0;
  GRID_STRIDE(e, L.m) {
    const uint32_t u = L.esrc[e], v = L.adj[e].x;
    if (label[u] < 0 && label[v] < 0) {
      const uint32_t cu = __ldcg(color + u);
      if (cu > __ldcg(color + v)) {
        atomicMax(color + v, cu);
        ch = 1;
      }
    }
  }
  if (__syncthreads_or(ch) && threadIdx.x == 0) *changed = 1;
}
__global__ void k_scc_roots(const int32_t* __restrict__ label, const uint32_t* __restrict__ color,
                            uint8_t* __restrict__ vis, int64_t n) {
  GRID_STRIDE(v, n) if (label[v] < 0 && color[v] == (uint32_t)v) vis[v] = 1;
}
// backward closure inside each colour: u joins if it reaches a member
__global__ void k_scc_bw(LG L, const int32_t* __restrict__ label, const uint32_t* __restrict__ color,
                         uint8_t* __restrict__ vis, int* __restrict__ changed) {
  int ch = 0;
  GRID_STRIDE(e, L.m) {
    const uint32_t u = L.esrc[e], v = L.adj[e].x;
    if (label[u] < 0 && !vis[u] && vis[v] && color[u] == color[v]) {
      vis[u] = 1;
      ch = 1;
    }
  }
  if (__syncthreads_or(ch) && threadIdx.x == 0) *changed = 1;
}
__global__ void k_scc_assign(int32_t* __restrict__ label, const uint32_t* __restrict__ color,
                             const uint8_t* __restrict__ vis, int64_t n, unsigned long long* __restrict__ left) {
  unsigned long long c = 0;
  GRID_STRIDE(v, n) {
    if (label[v] < 0) {
      if (vis[v]) label[v] = (int32_t)color[v];
      else c++;
    }
  }
  c = warp_sum_u64(c);
  if (lane_id() == 0 && c) atomicAdd(left, c);
}
__global__ void k_scc_min(const int32_t* __restrict__ label, int32_t* __restrict__ smin, int64_t n) {
  GRID_STRIDE(v, n) atomicMin(smin + label[v], (int32_t)v);
}
__global__ void k_scc_final(const int32_t* __restrict__ label, const int32_t* __restrict__ smin,
                            int32_t* __restrict__ out, int64_t n) {
  GRID_STRIDE(v, n) out[v] = smin[label[v]];
}

// ---- partitioned contexts: every rank sweeps its share of the
// logical edges (a contiguous range of the edge list), the per-vertex state is
// reduced across ranks after every sweep and the rest runs identically on
// every rank's full copy.  The transports reduce u32 with MIN / SUM (dist.h),
// so a max is a min of complements and a u64 min two u32 mins (high word,
// then the low word among the copies holding the minimum high word).
__global__ void k_not_u32(uint32_t* __restrict__ a, int64_t n) { GRID_STRIDE(i, n) a[i] = ~a[i]; }
__global__ void k_u8_to_u32(const uint8_t* __restrict__ a, uint32_t* __restrict__ b, int64_t n) {
  GRID_STRIDE(i, n) b[i] = a[i];
}
__global__ void k_u32_to_u8(const uint32_t* __restrict__ b, uint8_t* __restrict__ a, int64_t n) {
  GRID_STRIDE(i, n) a[i] = b[i] ? 1 : 0;
}
__global__ void k_u64_hi(const unsigned long long* __restrict__ k, uint32_t* __restrict__ hi, int64_t n) {
  GRID_STRIDE(i, n) hi[i] = (uint32_t)(k[i] >> 32);
}
__global__ void k_u64_lo(const unsigned long long* __restrict__ k, const uint32_t* __restrict__ hi,
                         uint32_t* __restrict__ lo, int64_t n) {
  GRID_STRIDE(i, n) lo[i] = (uint32_t)(k[i] >> 32) == hi[i] ? (uint32_t)k[i] : 0xFFFFFFFFu;
}
__global__ void k_u64_join(unsigned long long* __restrict__ k, const uint32_t* __restrict__ hi,
                           const uint32_t* __restrict__ lo, int64_t n) {
  GRID_STRIDE(i, n) k[i] = ((unsigned long long)hi[i] << 32) | lo[i];
}
__global__ void k_iota_from(uint32_t* __restrict__ a, int64_t n, uint32_t base) {
  GRID_STRIDE(i, n) a[i] = base + (uint32_t)i;
}

static Exch rank_exch(Ctx* c) {
  Exch X;
  X.c = c;
  X.P = c->world;
  X.sim = false;
  return X;
}
// this rank's share [lo, hi) of the logical edges
static void rank_edges(Ctx* c, int64_t m, int64_t& lo, int64_t& hi) {
  lo = m * c->rank / c->world;
  hi = m * (c->rank + 1) / c->world;
}
// a u32 flag summed over the ranks
static int sum_flag(Exch& X, int* flag, cudaStream_t s) {
  X.allreduce({flag}, 1, Dt::U32, Op::SUM);
  int h = 0;
  CUDA_OK(cudaMemcpyAsync(&h, flag, 4, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  return h;
}

static void run_scc_dist(gx_graph* g, gx_run_info& info, LG L) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  RunState& r = g->rs;
  const int64_t n = L.n;
  Exch X = rank_exch(c);
  int64_t e0_, e1_;
  rank_edges(c, L.m, e0_, e1_);
  LG Lr = L;   // this rank's edges
  Lr.adj = L.adj + e0_;
  Lr.esrc = L.esrc + e0_;
  Lr.m = e1_ - e0_;
  r.label.alloc(c, sizeof(int32_t) * n);
  r.label2.alloc(c, sizeof(int32_t) * n);
  r.comp.alloc(c, sizeof(uint32_t) * n);
  r.changed.alloc(c, 64);
  DBuf vis, vis32;
  vis.alloc(c, n);
  vis32.alloc(c, sizeof(uint32_t) * n);
  int32_t* label = r.label.as<int32_t>();
  uint32_t* color = r.comp.as<uint32_t>();
  int* changed = r.changed.as<int>();
  unsigned long long* left = reinterpret_cast<unsigned long long*>(r.changed.as<char>() + 8);
  const int gn = grid_for(c, n), ge = grid_for(c, std::max<int64_t>(Lr.m, 1));
  cudaEvent_t ev0, ev1;
  CUDA_OK(cudaEventCreate(&ev0));
  CUDA_OK(cudaEventCreate(&ev1));
  CUDA_OK(cudaEventRecord(ev0, s));
  CUDA_OK(cudaMemsetAsync(label, 0xFF, sizeof(int32_t) * n, s));
  int launches = 0, rounds = 0;
  int64_t edges = 0;
  while (true) {
    k_scc_color_init<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n);
    launches++;
    for (;;) {   // forward max-colour rounds: this rank's edges, then the max over the ranks
      CUDA_OK(cudaMemsetAsync(changed, 0, 4, s));
      if (Lr.m) k_scc_fw<<<ge, 256, 0, s>>>(Lr, label, color, changed);
      k_not_u32<<<gn, 256, 0, s>>>(color, n);
      X.allreduce({color}, n, Dt::U32, Op::MIN);
      k_not_u32<<<gn, 256, 0, s>>>(color, n);
      launches += 3;
      rounds++;
      edges += Lr.m;
      if (!sum_flag(X, changed, s)) break;
    }
    k_scc_roots<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n);
    launches++;
    for (;;) {   // backward closure rounds: this rank's edges, then the OR over the ranks
      CUDA_OK(cudaMemsetAsync(changed, 0, 4, s));
      if (Lr.m) k_scc_bw<<<ge, 256, 0, s>>>(Lr, label, color, vis.as<uint8_t>(), changed);
      k_u8_to_u32<<<gn, 256, 0, s>>>(vis.as<uint8_t>(), vis32.as<uint32_t>(), n);
      X.allreduce({vis32.p}, n, Dt::U32, Op::SUM);
      k_u32_to_u8<<<gn, 256, 0, s>>>(vis32.as<uint32_t>(), vis.as<uint8_t>(), n);
      launches += 3;
      rounds++;
      edges += Lr.m;
      if (!sum_flag(X, changed, s)) break;
    }
    unsigned long long hl = 0;   // labels and vis agree on every rank: so does the count
    CUDA_OK(cudaMemsetAsync(left, 0, 8, s));
    k_scc_assign<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n, left);
    launches++;
    CUDA_OK(cudaMemcpyAsync(&hl, left, 8, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (hl == 0) break;
  }
  DBuf smin;
  smin.alloc(c, sizeof(int32_t) * n);
  CUDA_OK(cudaMemsetAsync(smin.p, 0x7F, sizeof(int32_t) * n, s));
  k_scc_min<<<gn, 256, 0, s>>>(label, smin.as<int32_t>(), n);
  k_scc_final<<<gn, 256, 0, s>>>(label, smin.as<int32_t>(), r.label2.as<int32_t>(), n);
  launches += 2;
  CUDA_OK(cudaEventRecord(ev1, s));
  CUDA_OK(cudaEventSynchronize(ev1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, ev0, ev1));
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 16;
  info.kernel_launches = launches;
  r.have[GX_SCC] = true;
}

void run_scc(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  LG L = logical(g);
  RunState& r = g->rs;
  const int64_t n = L.n;
  GX_CHECK_ARG(n > 0, "empty graph");
  if (c->world > 1) {
    run_scc_dist(g, info, L);
    return;
  }
  r.label.alloc(c, sizeof(int32_t) * n);
  r.label2.alloc(c, sizeof(int32_t) * n);
  r.comp.alloc(c, sizeof(uint32_t) * n);
  r.changed.alloc(c, 64);
  DBuf vis;
  vis.alloc(c, n);
  int32_t* label = r.label.as<int32_t>();
  uint32_t* color = r.comp.as<uint32_t>();
  int* changed = r.changed.as<int>();
  unsigned long long* left = reinterpret_cast<unsigned long long*>(r.changed.as<char>() + 8);
  const int gn = grid_for(c, n), ge = grid_for(c, std::max<int64_t>(L.m, 1));
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(label, 0xFF, sizeof(int32_t) * n, s));
  int launches = 0, rounds = 0;
  int64_t edges = 0;
  while (true) {
    k_scc_color_init<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n);
    launches++;
    for (;;) {
      int h = 0;
      CUDA_OK(cudaMemsetAsync(changed, 0, 4, s));
      k_scc_fw<<<ge, 256, 0, s>>>(L, label, color, changed);
      launches++;
      rounds++;
      edges += L.m;
      CUDA_OK(cudaMemcpyAsync(&h, changed, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (!h) break;
    }
    k_scc_roots<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n);
    launches++;
    for (;;) {
      int h = 0;
      CUDA_OK(cudaMemsetAsync(changed, 0, 4, s));
      k_scc_bw<<<ge, 256, 0, s>>>(L, label, color, vis.as<uint8_t>(), changed);
      launches++;
      rounds++;
      edges += L.m;
      CUDA_OK(cudaMemcpyAsync(&h, changed, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (!h) break;
    }
    unsigned long long hl = 0;
    CUDA_OK(cudaMemsetAsync(left, 0, 8, s));
    k_scc_assign<<<gn, 256, 0, s>>>(label, color, vis.as<uint8_t>(), n, left);
    launches++;
    CUDA_OK(cudaMemcpyAsync(&hl, left, 8, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (hl == 0) break;
  }
  DBuf smin;
  smin.alloc(c, sizeof(int32_t) * n);
  CUDA_OK(cudaMemsetAsync(smin.p, 0x7F, sizeof(int32_t) * n, s));
  k_scc_min<<<gn, 256, 0, s>>>(label, smin.as<int32_t>(), n);
  k_scc_final<<<gn, 256, 0, s>>>(label, smin.as<int32_t>(), r.label2.as<int32_t>(), n);
  launches += 2;
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 16;  // esrc 4 + {dst,w} 8 + 2 label/colour gathers
  info.kernel_launches = launches;
  r.have[GX_SCC] = true;
}

// ---------------------------------------------------------------- MST
// min (weight, edge) key of every component over the active edges (all edges
// in round 1, then the compacted cross-component list): the current best is
// read first, so the atomic is skipped for the (late-round: nearly all) keys
// that cannot win -- Boruvka's later rounds hit a handful of components and
// unconditional atomics on them serialise at L2
__global__ void k_mst_best(LG L, const uint32_t* __restrict__ act, int64_t na, const uint32_t* __restrict__ comp,
                           unsigned long long* __restrict__ best, int* __restrict__ any) {
  int a = 0;
  GRID_STRIDE(i, na) {
    const uint32_t e = act ? act[i] : (uint32_t)i;
    const uint32_t u = L.esrc[e];
    const uint2 ed = L.adj[e];
    const uint32_t cu = comp[u], cv = comp[ed.x];
    if (cu != cv) {
      const unsigned long long key = ((unsigned long long)ed.y << 32) | (unsigned long long)e;
      if (key < __ldcg(best + cu)) atomicMin(best + cu, key);
      if (key < __ldcg(best + cv)) atomicMin(best + cv, key);
      a = 1;
    }
  }
  if (__syncthreads_or(a) && threadIdx.x == 0) *any = 1;
}
// the edges still joining two components after the round's merges
struct MstCross {
  const uint32_t* esrc;
  const uint2* adj;
  const uint32_t* comp;
  __device__ __forceinline__ bool operator()(const uint32_t& e) const {
    return comp[esrc[e]] != comp[adj[e].x];
  }
};
__global__ void k_mst_hook(LG L, const uint32_t* __restrict__ comp, const unsigned long long* __restrict__ best,
                           uint32_t* __restrict__ parent, int64_t n) {
  GRID_STRIDE(cc, n) {
    parent[cc] = (uint32_t)cc;
    if (comp[cc] != (uint32_t)cc || best[cc] == ~0ull) continue;
    const uint32_t e = (uint32_t)(best[cc] & 0xffffffffull);
    const uint32_t cu = comp[L.esrc[e]], cv = comp[L.adj[e].x];
    parent[cc] = cu == (uint32_t)cc ? cv : cu;
  }
}
__global__ void k_mst_resolve(const uint32_t* __restrict__ comp, const unsigned long long* __restrict__ best,
                              uint32_t* __restrict__ parent, int64_t n, unsigned long long* __restrict__ wsum) {
  unsigned long long w = 0;
  GRID_STRIDE(cc, n) {
    if (comp[cc] != (uint32_t)cc || best[cc] == ~0ull) continue;
    const uint32_t o = parent[cc];
    const bool mutual = parent[o] == (uint32_t)cc;
    if (!(mutual && (uint32_t)cc < o)) w += best[cc] >> 32;   // each chosen edge once
  }
  w = warp_sum_u64(w);
  if (lane_id() == 0 && w) atomicAdd(wsum, w);
}
__global__ void k_mst_root(const uint32_t* __restrict__ comp, const unsigned long long* __restrict__ best,
                           uint32_t* __restrict__ parent, int64_t n) {
  GRID_STRIDE(cc, n) {
    if (comp[cc] != (uint32_t)cc || best[cc] == ~0ull) continue;
    const uint32_t o = parent[cc];
    if (parent[o] == (uint32_t)cc && (uint32_t)cc < o) parent[cc] = (uint32_t)cc;
  }
}
__global__ void k_mst_jump(uint32_t* __restrict__ parent, int64_t n, int* __restrict__ changed) {
  int ch = 0;
  GRID_STRIDE(cc, n) {
    const uint32_t p = parent[cc], pp = parent[p];
    if (p != pp) {
      parent[cc] = pp;
      ch = 1;
    }
  }
  if (__syncthreads_or(ch) && threadIdx.x == 0) *changed = 1;
}
__global__ void k_mst_relabel(uint32_t* __restrict__ comp, const uint32_t* __restrict__ parent, int64_t n) {
  GRID_STRIDE(v, n) comp[v] = parent[comp[v]];
}
__global__ void k_iota_u32(uint32_t* __restrict__ a, int64_t n) { GRID_STRIDE(i, n) a[i] = (uint32_t)i; }

// Borůvka on a partitioned context: each rank proposes the lightest edge of
// every component over ITS active edges, the proposals are min-reduced over the
// ranks (two u32 mins: weight word, then the edge id among the copies holding
// the minimum weight), and hooking / pointer jumping / relabelling run
// identically on every rank's full copy; each rank compacts its own edges
static void run_mst_dist(gx_graph* g, gx_run_info& info, LG L) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  RunState& r = g->rs;
  const int64_t n = L.n;
  Exch X = rank_exch(c);
  int64_t e0_, e1_;
  rank_edges(c, L.m, e0_, e1_);
  r.comp.alloc(c, sizeof(uint32_t) * n);
  r.mst_best.alloc(c, sizeof(unsigned long long) * n);
  r.changed.alloc(c, 64);
  DBuf parent, hi, lo;
  parent.alloc(c, sizeof(uint32_t) * n);
  hi.alloc(c, sizeof(uint32_t) * n);
  lo.alloc(c, sizeof(uint32_t) * n);
  uint32_t* comp = r.comp.as<uint32_t>();
  unsigned long long* best = r.mst_best.as<unsigned long long>();
  int* flag = r.changed.as<int>();
  unsigned long long* wsum = reinterpret_cast<unsigned long long*>(r.changed.as<char>() + 8);
  const int gn = grid_for(c, n);
  cudaEvent_t ev0, ev1;
  CUDA_OK(cudaEventCreate(&ev0));
  CUDA_OK(cudaEventCreate(&ev1));
  CUDA_OK(cudaEventRecord(ev0, s));
  k_iota_u32<<<gn, 256, 0, s>>>(comp, n);
  CUDA_OK(cudaMemsetAsync(wsum, 0, 8, s));
  int launches = 1, rounds = 0;
  int64_t edges = 0;
  DBuf act[2], nsel, stmp;
  int64_t na = e1_ - e0_;
  act[0].alloc(c, sizeof(uint32_t) * std::max<int64_t>(na, 1));
  act[1].alloc(c, sizeof(uint32_t) * std::max<int64_t>(na, 1));
  nsel.alloc(c, 8);
  if (na) k_iota_from<<<grid_for(c, na), 256, 0, s>>>(act[0].as<uint32_t>(), na, (uint32_t)e0_);
  int cur = 0;
  while (true) {
    CUDA_OK(cudaMemsetAsync(best, 0xFF, sizeof(unsigned long long) * n, s));
    CUDA_OK(cudaMemsetAsync(flag, 0, 4, s));
    if (na)
      k_mst_best<<<grid_for(c, na), 256, 0, s>>>(L, act[cur].as<uint32_t>(), na, comp, best, flag);
    k_u64_hi<<<gn, 256, 0, s>>>(best, hi.as<uint32_t>(), n);
    X.allreduce({hi.p}, n, Dt::U32, Op::MIN);
    k_u64_lo<<<gn, 256, 0, s>>>(best, hi.as<uint32_t>(), lo.as<uint32_t>(), n);
    X.allreduce({lo.p}, n, Dt::U32, Op::MIN);
    k_u64_join<<<gn, 256, 0, s>>>(best, hi.as<uint32_t>(), lo.as<uint32_t>(), n);
    edges += na;
    rounds++;
    launches += 4;
    if (!sum_flag(X, flag, s)) break;
    k_mst_hook<<<gn, 256, 0, s>>>(L, comp, best, parent.as<uint32_t>(), n);
    k_mst_resolve<<<gn, 256, 0, s>>>(comp, best, parent.as<uint32_t>(), n, wsum);
    k_mst_root<<<gn, 256, 0, s>>>(comp, best, parent.as<uint32_t>(), n);
    launches += 3;
    for (;;) {
      int ch = 0;
      CUDA_OK(cudaMemsetAsync(flag, 0, 4, s));
      k_mst_jump<<<gn, 256, 0, s>>>(parent.as<uint32_t>(), n, flag);
      launches++;
      CUDA_OK(cudaMemcpyAsync(&ch, flag, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (!ch) break;
    }
    k_mst_relabel<<<gn, 256, 0, s>>>(comp, parent.as<uint32_t>(), n);
    launches++;
    MstCross pred{L.esrc, L.adj, comp};
    size_t tb = 0;
    const uint32_t* al = act[cur].as<uint32_t>();
    CUDA_OK(cub::DeviceSelect::If(nullptr, tb, al, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), std::max<int64_t>(na, 1), pred, s));
    stmp.alloc(c, tb);
    int64_t hn = 0;
    if (na) {
      CUDA_OK(cub::DeviceSelect::If(stmp.p, tb, al, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), na, pred, s));
      launches++;
      CUDA_OK(cudaMemcpyAsync(&hn, nsel.p, 8, cudaMemcpyDeviceToHost, s));
    }
    CUDA_OK(cudaStreamSynchronize(s));
    cur ^= 1;
    na = hn;
  }
  unsigned long long W = 0;   // the chosen edges agree on every rank: so does the weight
  CUDA_OK(cudaMemcpyAsync(&W, wsum, 8, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaEventRecord(ev1, s));
  CUDA_OK(cudaEventSynchronize(ev1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, ev0, ev1));
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  r.mst_weight = W;
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 20;
  info.kernel_launches = launches;
  r.have[GX_MST] = true;
}

void run_mst(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  LG L = logical(g);
  RunState& r = g->rs;
  const int64_t n = L.n;
  GX_CHECK_ARG(n > 0, "empty graph");
  GX_CHECK_ARG(L.m < (int64_t(1) << 32), "too many edges for 32-bit edge keys");
  if (c->world > 1) {
    run_mst_dist(g, info, L);
    return;
  }
  r.comp.alloc(c, sizeof(uint32_t) * n);
  r.mst_best.alloc(c, sizeof(unsigned long long) * n);
  r.changed.alloc(c, 64);
  DBuf parent;
  parent.alloc(c, sizeof(uint32_t) * n);
  uint32_t* comp = r.comp.as<uint32_t>();
  unsigned long long* best = r.mst_best.as<unsigned long long>();
  int* flag = r.changed.as<int>();
  unsigned long long* wsum = reinterpret_cast<unsigned long long*>(r.changed.as<char>() + 8);
  const int gn = grid_for(c, n);
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  k_iota_u32<<<gn, 256, 0, s>>>(comp, n);
  CUDA_OK(cudaMemsetAsync(wsum, 0, 8, s));
  int launches = 1, rounds = 0;
  int64_t edges = 0;
  // active-edge lists (cub::DeviceSelect keeps edge order): round r scans only
  // the edges that still join two components
  DBuf act[2], nsel, stmp;
  int64_t na = L.m;
  const uint32_t* al = nullptr;
  int cur = 0;
  while (true) {
    int h = 0;
    CUDA_OK(cudaMemsetAsync(best, 0xFF, sizeof(unsigned long long) * n, s));
    CUDA_OK(cudaMemsetAsync(flag, 0, 4, s));
    k_mst_best<<<grid_for(c, std::max<int64_t>(na, 1)), 256, 0, s>>>(L, al, na, comp, best, flag);
    edges += na;
    rounds++;
    launches++;
    CUDA_OK(cudaMemcpyAsync(&h, flag, 4, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (!h) break;
    k_mst_hook<<<gn, 256, 0, s>>>(L, comp, best, parent.as<uint32_t>(), n);
    k_mst_resolve<<<gn, 256, 0, s>>>(comp, best, parent.as<uint32_t>(), n, wsum);
    k_mst_root<<<gn, 256, 0, s>>>(comp, best, parent.as<uint32_t>(), n);
    launches += 3;
    for (;;) {
      int ch = 0;
      CUDA_OK(cudaMemsetAsync(flag, 0, 4, s));
      k_mst_jump<<<gn, 256, 0, s>>>(parent.as<uint32_t>(), n, flag);
      launches++;
      CUDA_OK(cudaMemcpyAsync(&ch, flag, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (!ch) break;
    }
    k_mst_relabel<<<gn, 256, 0, s>>>(comp, parent.as<uint32_t>(), n);
    launches++;
    // compact the cross-component edges for the next round
    if (!act[0].p) {
      act[0].alloc(c, sizeof(uint32_t) * std::max<int64_t>(L.m, 1));
      act[1].alloc(c, sizeof(uint32_t) * std::max<int64_t>(L.m, 1));
      nsel.alloc(c, 8);
    }
    MstCross pred{L.esrc, L.adj, comp};
    size_t tb = 0;
    if (al) {
      CUDA_OK(cub::DeviceSelect::If(nullptr, tb, al, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), na, pred, s));
    } else {
      cub::CountingInputIterator<uint32_t> all(0);
      CUDA_OK(cub::DeviceSelect::If(nullptr, tb, all, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), na, pred, s));
    }
    stmp.alloc(c, tb);
    if (al) {
      CUDA_OK(cub::DeviceSelect::If(stmp.p, tb, al, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), na, pred, s));
    } else {
      cub::CountingInputIterator<uint32_t> all(0);
      CUDA_OK(cub::DeviceSelect::If(stmp.p, tb, all, act[cur ^ 1].as<uint32_t>(), nsel.as<int64_t>(), na, pred, s));
    }
    launches++;
    int64_t hn = 0;
    CUDA_OK(cudaMemcpyAsync(&hn, nsel.p, 8, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    cur ^= 1;
    al = act[cur].as<uint32_t>();
    na = hn;
  }
  unsigned long long W = 0;
  CUDA_OK(cudaMemcpyAsync(&W, wsum, 8, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  r.mst_weight = W;
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 20;  // esrc 4 + {dst,w} 8 + 2 comp gathers
  info.kernel_launches = launches;
  r.have[GX_MST] = true;
}

// ---------------------------------------------------------------- BC
// forward: warp per frontier vertex; a head joins level L+1 by CAS and
// accumulates sigma from every level-L predecessor (P@14089).
__global__ void k_bc_fwd(LG L, const int32_t* __restrict__ q, int64_t q0, int64_t q1, int32_t lvl,
                         int32_t* __restrict__ level, double* __restrict__ sigma, int32_t* __restrict__ qout,
                         unsigned int* __restrict__ qtail) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = q0 + warp; i < q1; i += nw) {
    const int32_t u = q[i];
    const double su = sigma[u];
    for (uint32_t e = L.rp[u] + lane_id(); e < L.rp[u + 1]; e += 32) {
      const uint32_t w = L.adj[e].x;
      int32_t lw = __ldcg(level + w);
      if (lw < 0) {
        if (atomicCAS(level + w, -1, lvl + 1) == -1) {
          const unsigned pos = atomicAdd(qtail, 1u);
          qout[pos] = (int32_t)w;
        }
        lw = lvl + 1;
      }
      if (lw == lvl + 1) atomicAdd(sigma + w, su);
    }
  }
}
// backward: delta(v) = sigma_v * sum_{v->w, level w = level v + 1} (1 + delta_w) / sigma_w  (Eq 1).
// Every vertex stores coef(v) = (1 + delta_v) / sigma_v once, when its own
// level is processed, so a successor costs 2 gathers (level, coef) instead of
// 3 (level, delta, sigma); the fp64 operations are the same, in the same order.
__global__ void k_bc_bwd(LG L, const int32_t* __restrict__ q, int64_t q0, int64_t q1, int32_t lvl, int32_t src,
                         const int32_t* __restrict__ level, const double* __restrict__ sigma, double* __restrict__ coef,
                         double* __restrict__ bc) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = q0 + warp; i < q1; i += nw) {
    const int32_t v = q[i];
    double acc = 0.0;
    for (uint32_t e = L.rp[v] + lane_id(); e < L.rp[v + 1]; e += 32) {
      const uint32_t w = L.adj[e].x;
      if (level[w] == lvl + 1) acc += coef[w];
    }
    const double sv = sigma[v];
    acc = warp_sum_f64(acc) * sv;
    if (lane_id() == 0) {
      coef[v] = (1.0 + acc) / sv;
      if (v != src) bc[v] += acc;   // Eq 2
    }
  }
}

// ---- batched Brandes: BCB sources at a time, per-vertex state interleaved
// ([v][b]: levels 16 B, sigma / coef / delta 32 B each), so one sector gather
// of a neighbour serves the whole batch and a vertex's edges are read once per
// level at which any source of the batch reaches it.  Per source the
// arithmetic is that of k_bc_fwd / k_bc_bwd: sigma sums are exact integers
// (order-free), each coef / delta is the same lane-strided sum + warp
// reduction, and bc[v] adds the batch's deltas in source order at the end.
constexpr int BCB = 4;

__global__ void k_bcb_seed(const int32_t* __restrict__ src, int nb, int32_t* __restrict__ level4,
                           double* __restrict__ sigma4, int32_t* __restrict__ qlev) {
  const int b = threadIdx.x;
  if (b < nb) {
    const int32_t s = src[b];
    level4[(int64_t)s * BCB + b] = 0;
    sigma4[(int64_t)s * BCB + b] = 1.0;
    qlev[s] = 0;
  }
}

__global__ void k_bcb_fwd(LG L, const int32_t* __restrict__ q, int64_t q0, int64_t q1, int32_t lvl,
                          int32_t* __restrict__ level4, double* __restrict__ sigma4, int32_t* __restrict__ qlev,
                          int32_t* __restrict__ qout, unsigned int* __restrict__ qtail) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = q0 + warp; i < q1; i += nw) {
    const int32_t u = q[i];
    const int4 lu = *reinterpret_cast<const int4*>(level4 + (int64_t)u * BCB);
    const int lus[BCB] = {lu.x, lu.y, lu.z, lu.w};
    double su[BCB];
    unsigned m = 0;
#pragma unroll
    for (int b = 0; b < BCB; b++) {
      if (lus[b] == lvl) m |= 1u << b;
      su[b] = sigma4[(int64_t)u * BCB + b];
    }
    for (uint32_t e = L.rp[u] + lane_id(); e < L.rp[u + 1]; e += 32) {
      const uint32_t w = L.adj[e].x;
      int32_t* lw4 = level4 + (int64_t)w * BCB;
      const int4 lw = __ldcg(reinterpret_cast<const int4*>(lw4));
      const int lws[BCB] = {lw.x, lw.y, lw.z, lw.w};
      bool claimed = false;
#pragma unroll
      for (int b = 0; b < BCB; b++) {
        if (!(m >> b & 1u)) continue;
        int l = lws[b];
        if (l < 0) {
          if (atomicCAS(lw4 + b, -1, lvl + 1) == -1) claimed = true;
          l = lvl + 1;   // a failed CAS lost to this level's other writer
        }
        if (l == lvl + 1) atomicAdd(sigma4 + (int64_t)w * BCB + b, su[b]);
      }
      if (claimed && atomicExch(qlev + w, lvl + 1) != lvl + 1) qout[atomicAdd(qtail, 1u)] = (int32_t)w;
    }
  }
}

__global__ void k_bcb_bwd(LG L, const int32_t* __restrict__ q, int64_t q0, int64_t q1, int32_t lvl,
                          const int32_t* __restrict__ level4, const double* __restrict__ sigma4,
                          double* __restrict__ coef4, double* __restrict__ delta4) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = q0 + warp; i < q1; i += nw) {
    const int32_t v = q[i];
    const int4 lv = *reinterpret_cast<const int4*>(level4 + (int64_t)v * BCB);
    const int lvs[BCB] = {lv.x, lv.y, lv.z, lv.w};
    unsigned m = 0;
#pragma unroll
    for (int b = 0; b < BCB; b++)
      if (lvs[b] == lvl) m |= 1u << b;
    double acc[BCB] = {0.0, 0.0, 0.0, 0.0};
    for (uint32_t e = L.rp[v] + lane_id(); e < L.rp[v + 1]; e += 32) {
      const uint32_t w = L.adj[e].x;
      const int4 lw = *reinterpret_cast<const int4*>(level4 + (int64_t)w * BCB);
      const int lws[BCB] = {lw.x, lw.y, lw.z, lw.w};
      unsigned hit = 0;
#pragma unroll
      for (int b = 0; b < BCB; b++)
        if ((m >> b & 1u) && lws[b] == lvl + 1) hit |= 1u << b;
      if (hit) {
        const double2 c01 = *reinterpret_cast<const double2*>(coef4 + (int64_t)w * BCB);
        const double2 c23 = *reinterpret_cast<const double2*>(coef4 + (int64_t)w * BCB + 2);
        const double cs[BCB] = {c01.x, c01.y, c23.x, c23.y};
#pragma unroll
        for (int b = 0; b < BCB; b++)
          if (hit >> b & 1u) acc[b] += cs[b];
      }
    }
#pragma unroll
    for (int b = 0; b < BCB; b++) {
      if (!(m >> b & 1u)) continue;   // warp-uniform
      const double sv = sigma4[(int64_t)v * BCB + b];
      const double d = warp_sum_f64(acc[b]) * sv;
      if (lane_id() == 0) {
        coef4[(int64_t)v * BCB + b] = (1.0 + d) / sv;
        delta4[(int64_t)v * BCB + b] = d;
      }
    }
  }
}

// Eq 2 for the batch: bc[v] += delta_b(v) for b in source order, v != s_b
__global__ void k_bcb_acc(const double* __restrict__ delta4, const int32_t* __restrict__ src, int nb, int64_t n,
                          double* __restrict__ bc) {
  GRID_STRIDE(v, n) {
    double x = bc[v];
    for (int b = 0; b < nb; b++)
      if ((int32_t)v != src[b]) x += delta4[v * BCB + b];
    bc[v] = x;
  }
}

static void run_bc_batched(gx_graph* g, const gx_run_opts& o, gx_run_info& info, LG L) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  RunState& r = g->rs;
  const int64_t n = L.n;
  r.bc.alloc(c, sizeof(double) * n);
  r.changed.alloc(c, 64);
  DBuf level4, sigma4, coef4, delta4, qlev, q, dsrc;
  level4.alloc(c, sizeof(int32_t) * BCB * n);
  sigma4.alloc(c, sizeof(double) * BCB * n);
  coef4.alloc(c, sizeof(double) * BCB * n);
  delta4.alloc(c, sizeof(double) * BCB * n);
  qlev.alloc(c, sizeof(int32_t) * n);
  q.alloc(c, sizeof(int32_t) * BCB * n);   // a vertex is queued at most once per level it has for some source
  dsrc.alloc(c, sizeof(int32_t) * BCB);
  unsigned int* qtail = r.changed.as<unsigned int>();
  const int gw = c->num_sms * 16;
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(r.bc.p, 0, sizeof(double) * n, s));
  int launches = 0, rounds = 0;
  int64_t edges = 0;
  for (int64_t s0 = 0; s0 < o.n_bc_sources; s0 += BCB) {
    const int nbat = (int)std::min<int64_t>(BCB, o.n_bc_sources - s0);
    int32_t hs[BCB];
    for (int b = 0; b < nbat; b++) hs[b] = (int32_t)o.bc_sources[s0 + b];
    std::vector<int32_t> q0v;
    for (int b = 0; b < nbat; b++)
      if (std::find(q0v.begin(), q0v.end(), hs[b]) == q0v.end()) q0v.push_back(hs[b]);
    CUDA_OK(cudaMemsetAsync(level4.p, 0xFF, sizeof(int32_t) * BCB * n, s));
    CUDA_OK(cudaMemsetAsync(qlev.p, 0xFF, sizeof(int32_t) * n, s));
    CUDA_OK(cudaMemsetAsync(sigma4.p, 0, sizeof(double) * BCB * n, s));
    CUDA_OK(cudaMemsetAsync(delta4.p, 0, sizeof(double) * BCB * n, s));
    CUDA_OK(cudaMemcpyAsync(dsrc.p, hs, sizeof(int32_t) * nbat, cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(q.p, q0v.data(), sizeof(int32_t) * q0v.size(), cudaMemcpyHostToDevice, s));
    const unsigned int tail0 = (unsigned int)q0v.size();
    CUDA_OK(cudaMemcpyAsync(qtail, &tail0, 4, cudaMemcpyHostToDevice, s));
    k_bcb_seed<<<1, 32, 0, s>>>(dsrc.as<int32_t>(), nbat, level4.as<int32_t>(), sigma4.as<double>(), qlev.as<int32_t>());
    launches++;
    std::vector<int64_t> off{0, (int64_t)q0v.size()};
    for (int32_t lvl = 0;; lvl++) {
      const int64_t a = off[lvl], b = off[lvl + 1];
      if (b == a) break;
      k_bcb_fwd<<<gw, 256, 0, s>>>(L, q.as<int32_t>(), a, b, lvl, level4.as<int32_t>(), sigma4.as<double>(),
                                   qlev.as<int32_t>(), q.as<int32_t>(), qtail);
      launches++;
      rounds++;
      unsigned int t = 0;
      CUDA_OK(cudaMemcpyAsync(&t, qtail, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      off.push_back(t);
    }
    const int32_t D = (int32_t)off.size() - 2;
    for (int32_t lvl = D; lvl >= 0; lvl--) {
      k_bcb_bwd<<<gw, 256, 0, s>>>(L, q.as<int32_t>(), off[lvl], off[lvl + 1], lvl, level4.as<int32_t>(),
                                   sigma4.as<double>(), coef4.as<double>(), delta4.as<double>());
      launches++;
    }
    k_bcb_acc<<<grid_for(c, n), 256, 0, s>>>(delta4.as<double>(), dsrc.as<int32_t>(), nbat, n, r.bc.as<double>());
    launches++;
    edges += 2 * L.m * nbat;   // per source, as the single-source path counts
  }
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 20;
  info.kernel_launches = launches;
  r.have[GX_BC] = true;
}

void run_bc(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  LG L = logical(g);
  RunState& r = g->rs;
  const int64_t n = L.n;
  GX_CHECK_ARG(n > 0, "empty graph");
  GX_CHECK_ARG(o.bc_sources != nullptr && o.n_bc_sources > 0, "BC needs bc_sources (reading R37)");
  for (int64_t i = 0; i < o.n_bc_sources; i++)
    GX_CHECK_ARG(o.bc_sources[i] >= 0 && o.bc_sources[i] < n, "BC source out of range");
  if (c->world > 1) {
    // partitioned context (SURVEY §8(e) "BC: source-parallel"): rank p takes the
    // sources p, p + P, p + 2P, ... on its full graph copy, then ONE
    // allreduce(sum) of the bc vector; every rank ends with the whole result
    std::vector<int64_t> mine;
    for (int64_t i = c->rank; i < o.n_bc_sources; i += c->world) mine.push_back(o.bc_sources[i]);
    gx_run_opts ol = o;
    ol.bc_sources = mine.data();
    ol.n_bc_sources = (int64_t)mine.size();
    r.bc.alloc(c, sizeof(double) * n);
    if (mine.empty()) {
      CUDA_OK(cudaMemsetAsync(r.bc.p, 0, sizeof(double) * n, s));
      info = gx_run_info{};
      info.converged = 1;
    } else {
      run_bc_batched(g, ol, info, L);
    }
    Exch X;
    X.c = c;
    X.P = c->world;
    X.sim = false;
    X.allreduce({r.bc.p}, n, Dt::F64, Op::SUM);
    CUDA_OK(cudaStreamSynchronize(s));
    r.have[GX_BC] = true;
    return;
  }
  if (!getenv("GX_BC_SINGLE")) {   // batched sources (default); GX_BC_SINGLE=1: one source at a time
    run_bc_batched(g, o, info, L);
    return;
  }
  r.level.alloc(c, sizeof(int32_t) * n);
  r.sigma.alloc(c, sizeof(double) * n);
  r.delta.alloc(c, sizeof(double) * n);
  r.bc.alloc(c, sizeof(double) * n);
  r.changed.alloc(c, 64);
  DBuf q;
  q.alloc(c, sizeof(int32_t) * n);
  unsigned int* qtail = r.changed.as<unsigned int>();
  const int gn = grid_for(c, n);
  const int gw = c->num_sms * 16;
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(r.bc.p, 0, sizeof(double) * n, s));
  int launches = 0, rounds = 0;
  int64_t edges = 0;
  for (int64_t si = 0; si < o.n_bc_sources; si++) {
    const int32_t src = (int32_t)o.bc_sources[si];
    CUDA_OK(cudaMemsetAsync(r.level.p, 0xFF, sizeof(int32_t) * n, s));
    CUDA_OK(cudaMemsetAsync(r.sigma.p, 0, sizeof(double) * n, s));
    CUDA_OK(cudaMemsetAsync(r.delta.p, 0, sizeof(double) * n, s));
    const int32_t zero = 0;
    const double one = 1.0;
    const unsigned int tail1 = 1;
    CUDA_OK(cudaMemcpyAsync(r.level.as<int32_t>() + src, &zero, 4, cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(r.sigma.as<double>() + src, &one, 8, cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(q.as<int32_t>(), &src, 4, cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(qtail, &tail1, 4, cudaMemcpyHostToDevice, s));
    std::vector<int64_t> off{0, 1};
    for (int32_t lvl = 0;; lvl++) {
      const int64_t q0 = off[lvl], q1 = off[lvl + 1];
      if (q1 == q0) break;
      k_bc_fwd<<<gw, 256, 0, s>>>(L, q.as<int32_t>(), q0, q1, lvl, r.level.as<int32_t>(), r.sigma.as<double>(),
                                  q.as<int32_t>(), qtail);
      launches++;
      rounds++;
      unsigned int t = 0;
      CUDA_OK(cudaMemcpyAsync(&t, qtail, 4, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      off.push_back(t);
    }
    // levels 0..D: off[l]..off[l+1]
    const int32_t D = (int32_t)off.size() - 2;
    for (int32_t lvl = D; lvl >= 0; lvl--) {   // level D: no successors, coef = 1 / sigma
      k_bc_bwd<<<gw, 256, 0, s>>>(L, q.as<int32_t>(), off[lvl], off[lvl + 1], lvl, src, r.level.as<int32_t>(),
                                  r.sigma.as<double>(), r.delta.as<double>(), r.bc.as<double>());
      launches++;
    }
    edges += 2 * L.m;  // upper bound: every reached row scanned forward and backward
  }
  (void)gn;
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = rounds;
  info.converged = 1;
  info.loop_ms = ms;
  info.edges_scanned = edges;
  info.bytes_model = edges * 20;
  info.kernel_launches = launches;
  r.have[GX_BC] = true;
}

}  // namespace gx
