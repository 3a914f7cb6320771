// sssp.cu -- SSSP sweeps.
//
// The paper's primary kernel is vertex-centric neighbour enumeration with a
// "main fixed-point loop repeatedly calling the primary kernel" (PAPER.md
// P@15381, P@40883).  Here each iteration relaxes the out-edges of the active
// slots with atomicMin (exact integer arithmetic, bit-exact with Dijkstra on
// G_L, Theorem E1), then runs the §3 shared-memory pass over the subgraph
// tiles, then the §2.4 confluence (P@28309) of replica groups.
//
// LB mapping (best exact kernel): frontier queues, one persistent grid;
//   heavy slots (out-degree > HEAVY_DEG) are split into HCHUNK-edge work
//   items fetched with one atomic per warp; light slots are taken 32 at a
//   time per warp and their edges are distributed over the lanes by a warp
//   prefix scan (every lane relaxes one edge per round: coalesced 8-byte
//   {col, w} loads, no divergence from degree skew).  Newly improved slots
//   are deduplicated with a 1-bit-per-slot bitmap (atomicOr) and appended with
//   warp-aggregated atomics.
// TPV mapping (the paper's thread-per-vertex, §2/§4 layouts): tpv.cu.
#include <algorithm>
#include <chrono>
#include <cmath>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "ktimer.h"
#include "sssp_common.cuh"

namespace gx {

// ---------------------------------------------------------------- helpers
// L2 residency: dist is the only vector gathered at
// random, so its loads / atomics carry evict_last; the edge stream, queues
// and row offsets carry evict_first.  Frontier dedupe uses 1-bit-per-slot
// bitmaps (2 MB at 16M slots, always L2 resident), double-buffered by
// iteration parity: iteration t sets bits of bm[(t+1)&1] and clears bm[t&1].
struct SsspAux {
  uint32_t* bm[2];             // "already in the next frontier" bitmaps
  const uint32_t* heavy;       // bitmap: out-degree > HEAVY_DEG
  int64_t nwords;
};

__device__ __forceinline__ void push_next(bool push, uint32_t v, const uint32_t* __restrict__ rp,
                                          const uint32_t* __restrict__ heavybm, SsspCtr* nxt,
                                          int32_t* __restrict__ lq_out, int32_t* __restrict__ hq_out,
                                          uint32_t* __restrict__ hb_out) {
  unsigned bal = __ballot_sync(FULL, push);
  if (!bal) return;
  const bool heavy = push && ((__ldg(heavybm + (v >> 5)) >> (v & 31)) & 1u);
  unsigned lb = __ballot_sync(FULL, push && !heavy);
  if (lb) {
    unsigned leader = __ffs(lb) - 1, base = 0;
    if (lane_id() == leader) base = atomicAdd(&nxt->lcount, (unsigned)__popc(lb));
    base = __shfl_sync(FULL, base, leader);
    if (push && !heavy) st_stream_i32(lq_out + base + __popc(lb & lanemask_lt()), (int32_t)v, l2_evict_first());
  }
  if (heavy) {
    uint32_t vdeg = rp[v + 1] - rp[v];
    unsigned long long add = (1ull << 32) | (unsigned long long)((vdeg + HCHUNK - 1) / HCHUNK);
    unsigned long long old = atomicAdd(&nxt->hpack, add);
    hq_out[old >> 32] = (int32_t)v;
    hb_out[old >> 32] = (uint32_t)(old & 0xffffffffull);
  }
}

// relax one edge given the (possibly stale, never smaller) current distance
// `cur` of its head; returns true iff the head must join the next frontier
__device__ __forceinline__ bool relax2(uint2 ed, uint32_t du, uint32_t cur, uint32_t* __restrict__ dist,
                                       uint32_t* __restrict__ bm_next, uint64_t pl) {
  uint32_t nd = du + ed.y;
  if (nd < du) nd = INF - 1;  // saturate (never the fixed point)
  if (nd < cur) {
    uint32_t old = atom_min_l2(dist + ed.x, nd, pl);
    if (nd < old) {
      uint32_t bit = 1u << (ed.x & 31);
      if (!(atom_or_l2(bm_next + (ed.x >> 5), bit, pl) & bit)) return true;
    }
  }
  return false;
}

__device__ __forceinline__ void clear_bitmap(uint32_t* bm, int64_t nwords) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nwords; i += (int64_t)gridDim.x * blockDim.x)
    bm[i] = 0u;
}

// ---------------------------------------------------------------- LB sweep
constexpr int SU = 4;  // edges in flight per lane per round

__global__ void __launch_bounds__(256) k_sssp_lb(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj,
                                                 uint32_t* __restrict__ dist, SsspAux ax,
                                                 SsspQueues qs, SsspState* __restrict__ st) {
  __shared__ unsigned long long sh[32];
  const unsigned t = st->iter;
  if (st->stop) return;
  const bool odd = t & 1;
  SsspCtr* cur = &st->ctr[t % 3];
  SsspCtr* nxt = &st->ctr[(t + 1) % 3];
  const int32_t* lq_in = odd ? qs.lq[1] : qs.lq[0];
  int32_t* lq_out = odd ? qs.lq[0] : qs.lq[1];
  const int32_t* hq_in = odd ? qs.hq[1] : qs.hq[0];
  const uint32_t* hb_in = odd ? qs.hb[1] : qs.hb[0];
  int32_t* hq_out = odd ? qs.hq[0] : qs.hq[1];
  uint32_t* hb_out = odd ? qs.hb[0] : qs.hb[1];
  const unsigned lcount = cur->lcount;
  const unsigned long long hp = cur->hpack;
  const unsigned hcount = (unsigned)(hp >> 32), hchunks = (unsigned)(hp & 0xffffffffull);
  const unsigned lane = lane_id();
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  uint32_t* bm_next = odd ? ax.bm[0] : ax.bm[1];
  clear_bitmap(odd ? ax.bm[1] : ax.bm[0], ax.nwords);
  unsigned long long my_edges = 0;

  // heavy slots: HCHUNK-edge work items
  while (true) {
    unsigned c = 0;
    if (lane == 0) c = atomicAdd(&cur->hcursor, 1u);
    c = __shfl_sync(FULL, c, 0);
    if (c >= hchunks) break;
    int lo = 0, hi = (int)hcount - 1;
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      if (hb_in[mid] <= c) lo = mid;
      else hi = mid - 1;
    }
    int32_t u = hq_in[lo];
    uint32_t du = ld_l2_u32(dist + u, pl);
    uint32_t a = rp[u] + (c - hb_in[lo]) * HCHUNK;
    uint32_t b = min(a + (uint32_t)HCHUNK, rp[u + 1]);
    for (uint32_t e0 = a; e0 < b; e0 += 32 * SU) {
      uint2 ed[SU];
      bool act[SU], push[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) {
        uint32_t e = e0 + q * 32 + lane;
        act[q] = e < b;
        ed[q] = act[q] ? ld_stream_u2(adj + e, pf) : make_uint2(0, 0);
      }
      uint32_t cv[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) cv[q] = act[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
      for (int q = 0; q < SU; q++) push[q] = act[q] && relax2(ed[q], du, cv[q], dist, bm_next, pl);
#pragma unroll
      for (int q = 0; q < SU; q++) push_next(push[q], ed[q].x, rp, ax.heavy, nxt, lq_out, hq_out, hb_out);
    }
    if (lane == 0) my_edges += b - a;
  }

  // light slots: 32 per warp, edges spread over lanes by a prefix scan
  while (true) {
    unsigned base = 0;
    if (lane == 0) base = atomicAdd(&cur->lcursor, 32u);
    base = __shfl_sync(FULL, base, 0);
    if (base >= lcount) break;
    unsigned idx = base + lane;
    uint32_t start = 0, deg = 0, du = 0;
    if (idx < lcount) {
      int32_t u = ld_stream_i32(lq_in + idx, pf);
      start = ld_stream_u32(rp + u, pf);
      deg = ld_stream_u32(rp + u + 1, pf) - start;
      du = ld_l2_u32(dist + u, pl);
    }
    uint32_t incl = warp_incl_scan_u32(deg);
    uint32_t excl = incl - deg;
    uint32_t total = __shfl_sync(FULL, incl, 31);
    for (uint32_t k0 = 0; k0 < total; k0 += 32 * SU) {
      uint2 ed[SU];
      uint32_t od[SU];
      bool act[SU], push[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) {
        uint32_t k = k0 + q * 32 + lane;
        int j = 0;
#pragma unroll
        for (int s = 16; s; s >>= 1) {
          uint32_t ex = __shfl_sync(FULL, excl, j + s);
          if (ex <= k) j += s;
        }
        uint32_t os = __shfl_sync(FULL, start, j);
        uint32_t oe = __shfl_sync(FULL, excl, j);
        od[q] = __shfl_sync(FULL, du, j);
        act[q] = k < total;
        ed[q] = act[q] ? ld_stream_u2(adj + os + (k - oe), pf) : make_uint2(0, 0);
      }
      uint32_t cv[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) cv[q] = act[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
      for (int q = 0; q < SU; q++) push[q] = act[q] && relax2(ed[q], od[q], cv[q], dist, bm_next, pl);
#pragma unroll
      for (int q = 0; q < SU; q++) push_next(push[q], ed[q].x, rp, ax.heavy, nxt, lq_out, hq_out, hb_out);
    }
    if (lane == 0) my_edges += total;
  }
  unsigned long long tot = block_sum_u64(my_edges, sh);
  if (threadIdx.x == 0 && tot) atomicAdd(&st->edges, tot);
}

// ---------------------------------------------------------------- §3 local pass
// One CTA per subgraph tile: member distances staged in shared memory,
// relaxed t times over the tile's local edges (P@32188-32416, reading R28),
// improvements written back with atomicMin and pushed to the next frontier.
__global__ void __launch_bounds__(256) k_sssp_local(const int32_t* __restrict__ tptr, const int32_t* __restrict__ tmem,
                                                    const int32_t* __restrict__ teptr, const uint2* __restrict__ tedges,
                                                    const int32_t* __restrict__ titers, int64_t ntiles,
                                                    const uint32_t* __restrict__ rp, uint32_t* __restrict__ dist,
                                                    SsspAux ax, SsspQueues qs, SsspState* __restrict__ st) {
  __shared__ uint32_t sd[256];
  const unsigned t = st->iter;
  if (st->stop) return;
  SsspCtr* nxt = &st->ctr[(t + 1) % 3];
  int32_t* lq_out = (t & 1) ? qs.lq[0] : qs.lq[1];
  int32_t* hq_out = (t & 1) ? qs.hq[0] : qs.hq[1];
  uint32_t* hb_out = (t & 1) ? qs.hb[0] : qs.hb[1];
  uint32_t* bm_next = (t & 1) ? ax.bm[0] : ax.bm[1];
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    int a = tptr[tile], nm = tptr[tile + 1] - a;
    int ea = teptr[tile], ne = teptr[tile + 1] - ea;
    for (int i = threadIdx.x; i < nm; i += blockDim.x) sd[i] = __ldcg(dist + tmem[a + i]);
    __syncthreads();
    int iters = titers[tile];
    for (int r = 0; r < iters; r++) {
      int ch = 0;
      for (int i = threadIdx.x; i < ne; i += blockDim.x) {
        uint2 p = tedges[ea + i];
        uint32_t src = p.x & 0xff, dst = (p.x >> 8) & 0xff, w = p.y;
        uint32_t du = sd[src];
        if (du != INF) {
          uint32_t nd = du + w;
          if (nd < du) nd = INF - 1;
          if (nd < sd[dst]) {
            atomicMin(&sd[dst], nd);
            ch = 1;
          }
        }
      }
      if (!__syncthreads_or(ch)) break;
    }
    for (int i0 = 0; i0 < nm; i0 += blockDim.x) {
      int i = i0 + threadIdx.x;
      bool push = false;
      uint32_t v = 0;
      if (i < nm) {
        v = (uint32_t)tmem[a + i];
        uint32_t nd = sd[i];
        if (nd < __ldcg(dist + v)) {
          uint32_t old = atomicMin(dist + v, nd);
          push = nd < old && !(atomicOr(bm_next + (v >> 5), 1u << (v & 31)) & (1u << (v & 31)));
        }
      }
      push_next(push, v, rp, ax.heavy, nxt, lq_out, hq_out, hb_out);
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- §2.4 merge
// One warp per confluence group.  The owner first re-pulls its in-edges (the
// Jacobi step a merge may have undone), then all
// copies take the mean (floor of the exact 64-bit mean, INF copies excluded,
// reading R19) or the min (GX_MERGE_MIN).  Copies that decrease re-enter the
// frontier.
__global__ void __launch_bounds__(256) k_sssp_merge(const int32_t* __restrict__ gptr, const int32_t* __restrict__ gslots,
                                                    const int32_t* __restrict__ ginptr, const uint2* __restrict__ gin,
                                                    int64_t ngroups, int merge_min, const uint32_t* __restrict__ rp,
                                                    uint32_t* __restrict__ dist, SsspAux ax,
                                                    SsspQueues qs, SsspState* __restrict__ st) {
  const unsigned t = st->iter;
  if (st->stop) return;
  SsspCtr* nxt = &st->ctr[(t + 1) % 3];
  int32_t* lq_out = (t & 1) ? qs.lq[0] : qs.lq[1];
  int32_t* hq_out = (t & 1) ? qs.hq[0] : qs.hq[1];
  uint32_t* hb_out = (t & 1) ? qs.hb[0] : qs.hb[1];
  uint32_t* bm_next = (t & 1) ? ax.bm[0] : ax.bm[1];
  const unsigned lane = lane_id();
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t gi = warp; gi < ngroups; gi += nw) {
    int a = gptr[gi], b = gptr[gi + 1];
    int32_t o = gslots[a];
    uint32_t best = INF;
    for (int e = ginptr[gi] + lane; e < ginptr[gi + 1]; e += 32) {
      uint2 iv = gin[e];
      uint32_t dp = dist[iv.x];
      if (dp != INF) best = min(best, dp + iv.y);
    }
    best = warp_min_u32(best);
    uint32_t own = min(dist[o], best);
    unsigned long long sum = 0;
    unsigned cnt = 0;
    uint32_t mn = INF;
    for (int i = a + lane; i < b; i += 32) {
      uint32_t val = (i == a) ? own : dist[gslots[i]];
      if (val != INF) {
        sum += val;
        cnt++;
      }
      mn = min(mn, val);
    }
    sum = warp_sum_u64(sum);
    cnt = __reduce_add_sync(FULL, cnt);
    mn = warp_min_u32(mn);
    uint32_t mval = merge_min ? mn : (cnt ? (uint32_t)(sum / cnt) : INF);
    for (int i0 = a; i0 < b; i0 += 32) {
      int i = i0 + lane;
      bool push = false;
      uint32_t s = 0;
      if (i < b) {
        s = (uint32_t)gslots[i];
        uint32_t old = dist[s];
        if (old != mval) {
          dist[s] = mval;
          push = mval < old && !(atomicOr(bm_next + (s >> 5), 1u << (s & 31)) & (1u << (s & 31)));
          if (mval > old) atomicAdd(&st->raised, 1u);
        }
      }
      push_next(push, s, rp, ax.heavy, nxt, lq_out, hq_out, hb_out);
    }
  }
}

__global__ void k_sssp_advance(SsspState* __restrict__ st, int max_iters) {
  if (st->stop) return;
  unsigned t = st->iter;
  SsspCtr* n1 = &st->ctr[(t + 1) % 3];
  SsspCtr* n2 = &st->ctr[(t + 2) % 3];
  n2->lcount = 0;
  n2->lcursor = 0;
  n2->hpack = 0;
  n2->hcursor = 0;
  st->active += (unsigned long long)n1->lcount + (n1->hpack >> 32);
  st->iter = t + 1;
  bool empty = n1->lcount == 0 && (n1->hpack >> 32) == 0;
  if (empty) st->stop = 1;           // converged
  else if ((int)(t + 1) >= max_iters) st->stop = 2;
}

__global__ void k_sssp_init(uint32_t* __restrict__ dist, const int32_t* __restrict__ slots, int nslots,
                            const uint32_t* __restrict__ rp, SsspQueues qs, SsspState* __restrict__ st) {
  // all copies of the source start at 0 (P@28609: copies begin equal)
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  for (int i = 0; i < nslots; i++) {
    int32_t s = slots[i];
    dist[s] = 0;
    uint32_t deg = rp[s + 1] - rp[s];
    if (deg > HEAVY_DEG) {
      unsigned long long old = st->ctr[0].hpack;
      st->ctr[0].hpack = old + ((1ull << 32) | ((deg + HCHUNK - 1) / HCHUNK));
      qs.hq[0][old >> 32] = s;
      qs.hb[0][old >> 32] = (uint32_t)(old & 0xffffffffull);
    } else {
      qs.lq[0][st->ctr[0].lcount++] = s;
    }
  }
  st->active = nslots;
}

// bitmap of slots whose out-degree exceeds HEAVY_DEG (push-time class test)
__global__ void k_heavy_bitmap(const uint32_t* __restrict__ rp, int64_t n, uint32_t* __restrict__ hb) {
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w * 32 < n; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = 0;
    for (int b = 0; b < 32; b++) {
      int64_t v = w * 32 + b;
      if (v < n && rp[v + 1] - rp[v] > HEAVY_DEG) bits |= 1u << b;
    }
    hb[w] = bits;
  }
}

// R36: max out-degree vertex of the canonical input, ties to the lowest id
__global__ void k_argmax_deg(const int64_t* __restrict__ rp, int64_t n, unsigned long long* __restrict__ out) {
  unsigned long long best = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    unsigned long long d = (unsigned long long)(rp[v + 1] - rp[v]);
    unsigned long long key = (d << 32) | (0xffffffffull - (unsigned long long)v);
    best = max(best, key);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) best = max(best, __shfl_xor_sync(FULL, best, o));
  if (lane_id() == 0) atomicMax(out, best);
}

int64_t default_source(gx_graph* g) {
  Ctx* c = g->ctx;
  DBuf b;
  b.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(b.p, 0, 8, c->stream));
  if (g->n) k_argmax_deg<<<grid_for(c, g->n), 256, 0, c->stream>>>(g->in_rp.as<int64_t>(), g->n,
                                                                   b.as<unsigned long long>());
  unsigned long long h = 0;
  CUDA_OK(cudaMemcpyAsync(&h, b.p, 8, cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  return (int64_t)(0xffffffffull - (h & 0xffffffffull));
}

// ---------------------------------------------------------------- driver
void run_sssp_tpv_iter(gx_graph* g, SsspQueues qs, SsspState* st, int& launches);  // tpv.cu (uses SsspAux via g)
void ensure_tpv(gx_graph* g);                                                    // tpv.cu

void run_sssp(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  int64_t src = o.source < 0 ? default_source(g) : o.source;
  GX_CHECK_ARG(g->n > 0, "empty graph");
  GX_CHECK_ARG(src >= 0 && src < g->n, "source out of range");
  if ((double)(g->n - 1) * (double)d.max_w >= 4294967295.0)
    GX_THROW(GX_E_UNSUPPORTED, "(n-1)*max(w) >= 2^32-1 would overflow uint32 distances");
  int mapping = o.mapping;
  if (mapping == GX_MAP_AUTO) mapping = (g->transformed && (g->knobs.coalesce || g->knobs.degree_norm)) ? GX_MAP_TPV : GX_MAP_LB;
  if (mapping == GX_MAP_TPV) ensure_tpv(g);
  int64_t ns = d.n_slots;
  r.dist.alloc(c, sizeof(uint32_t) * ns);
  const int64_t nwords = (ns + 31) / 32;
  r.mark.alloc(c, sizeof(uint32_t) * 3 * nwords);   // bm[0], bm[1], heavy
  for (int i = 0; i < 2; i++) {
    r.q[i].alloc(c, sizeof(int32_t) * ns);
    r.hq[i].alloc(c, sizeof(int32_t) * ns);
    r.hbase[i].alloc(c, sizeof(uint32_t) * ns);
  }
  r.st.alloc(c, sizeof(SsspState));
  SsspQueues qs;
  for (int i = 0; i < 2; i++) {
    qs.lq[i] = r.q[i].as<int32_t>();
    qs.hq[i] = r.hq[i].as<int32_t>();
    qs.hb[i] = r.hbase[i].as<uint32_t>();
  }
  SsspState* st = r.st.as<SsspState>();
  SsspAux ax;
  ax.bm[0] = r.mark.as<uint32_t>();
  ax.bm[1] = r.mark.as<uint32_t>() + nwords;
  ax.heavy = r.mark.as<uint32_t>() + 2 * nwords;
  ax.nwords = nwords;
  k_heavy_bitmap<<<grid_for(c, ns), 256, 0, s>>>(d.rp.as<uint32_t>(), ns, r.mark.as<uint32_t>() + 2 * nwords);
  CUDA_OK(cudaGetLastError());
  // source copies: owner slot + replica slots
  std::vector<int32_t> srcs;
  if (d.identity) {
    srcs.push_back((int32_t)src);
  } else {
    const SlotGraph& sg = g->sg;
    srcs.push_back(sg.owner_slot[src]);
    for (int64_t sl = 0; sl < sg.n_slots; sl++)
      if (sg.kind[sl] == REPLICA && sg.slot_to_orig[sl] == src) srcs.push_back((int32_t)sl);
  }
  DBuf dsrc;
  dsrc.alloc(c, sizeof(int32_t) * srcs.size());
  CUDA_OK(cudaMemcpyAsync(dsrc.p, srcs.data(), sizeof(int32_t) * srcs.size(), cudaMemcpyHostToDevice, s));

  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(r.dist.p, 0xFF, sizeof(uint32_t) * ns, s));
  CUDA_OK(cudaMemsetAsync(r.mark.p, 0, sizeof(uint32_t) * 2 * nwords, s));
  CUDA_OK(cudaMemsetAsync(r.st.p, 0, sizeof(SsspState), s));
  k_sssp_init<<<1, 32, 0, s>>>(r.dist.as<uint32_t>(), dsrc.as<int32_t>(), (int)srcs.size(), d.rp.as<uint32_t>(),
                               qs, st);
  CUDA_OK(cudaGetLastError());
  int launches = 4;

  int occ = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sssp_lb, 256, 0));
  int grid_lb = std::max(1, occ) * c->num_sms;
  int grid_local = (int)std::max<int64_t>(1, std::min<int64_t>(d.n_tiles, (int64_t)c->num_sms * 8));
  int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_groups + 7) / 8, (int64_t)c->num_sms * 8));
  bool merge_min = g->knobs.merge_op == GX_MERGE_MIN;

  KTimer kt(o.profile != 0, s);
  auto one_iter = [&](int& nl) {
    kt.begin();
    if (mapping == GX_MAP_TPV) {
      run_sssp_tpv_iter(g, qs, st, nl);
    } else {
      k_sssp_lb<<<grid_lb, 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), r.dist.as<uint32_t>(),
                                        ax, qs, st);
      nl++;
    }
    kt.end();
    if (d.n_tiles && g->knobs.smem) {
      k_sssp_local<<<grid_local, 256, 0, s>>>(d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(), d.t_eptr.as<int32_t>(),
                                              d.t_edges.as<uint2>(), d.t_iters.as<int32_t>(), d.n_tiles,
                                              d.rp.as<uint32_t>(), r.dist.as<uint32_t>(), ax, qs, st);
      nl++;
    }
    if (d.n_groups) {
      k_sssp_merge<<<grid_merge, 256, 0, s>>>(d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), d.g_in_ptr.as<int32_t>(),
                                              d.g_in.as<uint2>(), d.n_groups, merge_min ? 1 : 0, d.rp.as<uint32_t>(),
                                              r.dist.as<uint32_t>(), ax, qs, st);
      nl++;
    }
    k_sssp_advance<<<1, 1, 0, s>>>(st, o.max_iters);
    nl++;
  };

  int batch = std::max(1, o.check_every);
  cudaGraphExec_t gexec = nullptr;
  int per_batch_launches = 0;
  if (o.use_graphs && !o.profile) {
    cudaGraph_t graph;
    CUDA_OK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    for (int i = 0; i < batch; i++) one_iter(per_batch_launches);
    CUDA_OK(cudaStreamEndCapture(s, &graph));
    CUDA_OK(cudaGraphInstantiate(&gexec, graph, 0));
    CUDA_OK(cudaGraphDestroy(graph));
  }
  SsspState hst;
  int done_iters = 0;
  while (true) {
    if (gexec) {
      CUDA_OK(cudaGraphLaunch(gexec, s));
      launches += per_batch_launches;
    } else {
      for (int i = 0; i < batch; i++) one_iter(launches);
    }
    CUDA_OK(cudaGetLastError());
    done_iters += batch;
    CUDA_OK(cudaMemcpyAsync(&hst, st, sizeof(SsspState), cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (hst.stop) break;
  }
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  if (gexec) cudaGraphExecDestroy(gexec);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = (int32_t)hst.iter;
  info.converged = hst.stop == 1;
  info.loop_ms = ms;
  info.edges_scanned = (int64_t)hst.edges;
  info.vertices_active = (int64_t)hst.active;
  // bytes model: 12 B per scanned edge ({col,w} 8 + dist 4) +
  // 14 B per processed slot (row_ptr 8 + dist 4 + queue 2*... ~2)
  info.bytes_model = 12 * (int64_t)hst.edges + 14 * (int64_t)hst.active;
  info.kernel_launches = launches;
  info.sweep_launches = kt.launches();
  info.sweep_ms = kt.total_ms();
  info.sweep_bytes = info.bytes_model;
  r.have[GX_SSSP] = true;
}

}  // namespace gx
