// sssp.cu -- SSSP sweeps.
//
// The paper's primary kernel is vertex-centric neighbour enumeration with a
// "main fixed-point loop repeatedly calling the primary kernel" (PAPER.md
// P@15381, P@40883).  Here each iteration relaxes the out-edges of the active
// slots with atomic min (exact integer arithmetic, bit-exact with Dijkstra on
// G_L, Theorem E1), then runs the §3 shared-memory pass over the subgraph
// tiles, then the §2.4 confluence (P@28309) of replica groups.
//
// LB mapping (best exact kernel): the frontier is a bitmap.  Each warp
// compacts the set bits of 32 bitmap words (1024 slots) into shared memory
// and spreads the out-edges of 32 slots at a time over its lanes by a warp
// prefix scan (coalesced 8-byte {col, w} loads, no divergence from degree
// skew); slots with out-degree > HEAVY_DEG are relaxed from a static list of
// 1024-edge chunks.  A relaxation is fire-and-forget: red.min on dist and
// red.or on the next-frontier bitmap -- no return values, queues or counters,
// so nothing serialises on atomic round trips.  dist and the bitmaps carry
// L2 evict_last, the edge stream evict_first.
// TPV mapping (the paper's thread-per-vertex, §2/§4 layouts): tpv.cu.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>

#include <cooperative_groups.h>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "ktimer.h"
#include "sssp_common.cuh"
#include "dist.h"
#include "sell.cuh"
#include <cub/cub.cuh>
#include <cstdlib>
#include <cstring>

namespace gx {
namespace cg = cooperative_groups;

// ---------------------------------------------------------------- helpers
__device__ __forceinline__ bool bit_of(const uint32_t* __restrict__ bm, uint32_t v) {
  return (__ldcg(bm + (v >> 5)) >> (v & 31)) & 1u;
}

// relax one edge given the (possibly stale, never smaller within a sweep)
// distance `cur` of its head
__device__ __forceinline__ void relax_red(uint2 ed, uint32_t du, uint32_t cur, uint32_t* __restrict__ dist,
                                          uint32_t* __restrict__ bm_next, uint32_t& npush, uint64_t pl) {
  const uint32_t nd = sat_add(du, ed.y);   // R51
  if (nd < cur) {
    red_min_l2(dist + ed.x, nd, pl);
    red_or_l2(bm_next + (ed.x >> 5), 1u << (ed.x & 31), pl);
    npush++;
  }
}

// near-far relaxation: a head whose new distance is below tau joins the next
// frontier, otherwise the far pile (far_min tracks its smallest distance)
// word windows of the bits a thread pushed (frontier windows, SsspState)
struct Win {
  uint32_t nlo = 0xFFFFFFFFu, nhi = 0, flo = 0xFFFFFFFFu, fhi = 0;
};
__device__ __forceinline__ void relax_nf(uint2 ed, uint32_t du, uint32_t cur, uint32_t* __restrict__ dist,
                                         uint32_t* __restrict__ bm_next, uint32_t* __restrict__ far, uint32_t tau,
                                         uint32_t& far_min, uint32_t& npush, uint64_t pl, Win& wn) {
  const uint32_t nd = sat_add(du, ed.y);
  if (nd < cur) {
    red_min_l2(dist + ed.x, nd, pl);
    const uint32_t w = ed.x >> 5;
    if (nd < tau) {
      red_or_l2(bm_next + w, 1u << (ed.x & 31), pl);
      npush++;
      wn.nlo = min(wn.nlo, w);
      wn.nhi = max(wn.nhi, w);
    } else {
      if (far) red_or_l2(far + w, 1u << (ed.x & 31), pl);   // null: far pile by scan (sssp_split_dev)
      far_min = min(far_min, nd);
      wn.flo = min(wn.flo, w);
      wn.fhi = max(wn.fhi, w);
    }
  }
}

// the CTA's pushed-word windows into the state (one atomic of each per CTA;
// every thread of the CTA calls it): near pushes -> bm window *nw, far -> *fw
__device__ __forceinline__ void flush_windows(Win wn, unsigned* nlo, unsigned* nhi, unsigned* flo, unsigned* fhi) {
  __shared__ uint32_t s_w[4][32];
  wn.nlo = warp_min_u32(wn.nlo);
  wn.nhi = warp_max_u32(wn.nhi);
  wn.flo = warp_min_u32(wn.flo);
  wn.fhi = warp_max_u32(wn.fhi);
  const unsigned w = threadIdx.x >> 5, nwp = blockDim.x >> 5;
  if (lane_id() == 0) {
    s_w[0][w] = wn.nlo;
    s_w[1][w] = wn.nhi;
    s_w[2][w] = wn.flo;
    s_w[3][w] = wn.fhi;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    Win b;
    for (unsigned i = 0; i < nwp; i++) {
      b.nlo = min(b.nlo, s_w[0][i]);
      b.nhi = max(b.nhi, s_w[1][i]);
      b.flo = min(b.flo, s_w[2][i]);
      b.fhi = max(b.fhi, s_w[3][i]);
    }
    if (b.nlo <= b.nhi) {
      atomicMin(nlo, b.nlo);
      atomicMax(nhi, b.nhi);
    }
    if (b.flo <= b.fhi) {
      atomicMin(flo, b.flo);
      atomicMax(fhi, b.fhi);
    }
  }
  __syncthreads();
}

// Block-level reduction of a sweep's per-thread counters: one atomic of each
// kind per CTA (same-address atomics from every warp would serialise in L2).
// Every thread of the CTA must call it.
__device__ __forceinline__ void flush_counters(SsspState* st, unsigned t, unsigned long long edges,
                                               unsigned long long act, uint32_t push, uint32_t fmin,
                                               uint32_t* fdst = nullptr) {
  __shared__ unsigned long long s_e[32], s_a[32];
  __shared__ uint32_t s_p[32], s_m[32];
  edges = warp_sum_u64(edges);
  act = warp_sum_u64(act);
  push = __reduce_add_sync(FULL, push);
  fmin = warp_min_u32(fmin);
  const unsigned w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (lane_id() == 0) {
    s_e[w] = edges;
    s_a[w] = act;
    s_p[w] = push;
    s_m[w] = fmin;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long e = 0, a = 0;
    uint32_t p = 0, m = INF;
    for (unsigned i = 0; i < nw; i++) {
      e += s_e[i];
      a += s_a[i];
      p += s_p[i];
      m = min(m, s_m[i]);
    }
    if (e) atomicAdd(&st->edges, e);
    if (a) atomicAdd(&st->active[t % 3], (unsigned)a);
    if (p) atomicAdd(&st->pushed[t % 3], p);
    if (m != INF) atomicMin(fdst ? fdst : &st->far_min, m);
  }
}

__device__ __forceinline__ void clear_bitmap_range(uint32_t* bm, uint32_t lo, uint32_t hi) {
  if (lo > hi) return;
  for (int64_t i = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= (int64_t)hi; i += (int64_t)gridDim.x * blockDim.x)
    bm[i] = 0u;
}
__device__ __forceinline__ void clear_bitmap(uint32_t* bm, int64_t nwords) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nwords; i += (int64_t)gridDim.x * blockDim.x)
    bm[i] = 0u;
}

// ---------------------------------------------------------------- LB sweep
// measured (RMAT-24 exact, persistent loop, profiles/r1e/sssp_hint_variants.txt):
// row_ptr loads with L2 evict_first (the gathered dist keeps the L2) and 3
// edges in flight per lane: 5.04 -> 4.78 ms; SU 8: 5.8 ms; 5-6 CTAs/SM
// (__launch_bounds__ min blocks, spills): 5.9-9.8 ms.  Round 2, after the far
// pile by scan (profiles/r2/sssp_su_pipe_variants.txt): the software pipeline
// off and 5 edges in flight per lane: RMAT-24 4.06 -> 3.67 ms, uniform
// 16M/256M 4.05 -> 3.83, RMAT-22 1.93 -> 1.70 (SU 3 / 4 / 6 and the pipeline
// on are slower; 3 CTAs per SM 4.39)
#ifndef GX_SSSP_RP_EF
#define GX_SSSP_RP_EF 1
#endif
#ifndef GX_SSSP_SU
#define GX_SSSP_SU 5
#endif
constexpr int SU = GX_SSSP_SU;   // edges in flight per lane per round
#ifndef GX_SSSP_PIPE
#define GX_SSSP_PIPE 0
#endif
#ifndef GX_SSSP_TPB
#define GX_SSSP_TPB 256
#endif
constexpr int PERSIST_TPB = GX_SSSP_TPB;   // threads per CTA of the persistent loop
constexpr int SB_WARPS = PERSIST_TPB / 32 > 8 ? PERSIST_TPB / 32 : 8;   // warps per CTA (k_sssp_lb: 8)

// iteration t with near-far threshold tau; the far pile's minimum goes to fdst
__device__ __forceinline__ void sssp_lb_dev(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj,
                                            uint32_t* __restrict__ dist, const SsspAux& ax, SsspState* __restrict__ st,
                                            int64_t row_lo, int64_t row_hi, const unsigned t, const uint32_t tau,
                                            uint32_t* fdst, int32_t (*s_v)[1024], const int lh = 0,
                                            const int pp = 0, const unsigned far_slot = 0, const bool win = false) {
  // lh: 0 all edges; 1 light pass (light edges, frontier recorded in pend[pp]);
  // 2 heavy pass (heavy edges of pend[pp], pend[pp ^ 1] cleared for the next bucket)
  const uint32_t* __restrict__ bm_cur = lh == 2 ? ax.pend[pp] : ax.bm[t % 3];
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  uint32_t* pend_w = lh == 1 ? ax.pend[pp] : nullptr;
  // frontier windows (win: the persistent loop with st->win_on): scan and
  // clear only the words that can hold bits
  if (win) clear_bitmap_range(ax.bm[(t + 2) % 3], st->wlo[(t + 5) % 6], st->whi[(t + 5) % 6]);   // frontier t-1
  else clear_bitmap(ax.bm[(t + 2) % 3], ax.nwords);
  if (lh == 2) clear_bitmap(ax.pend[pp ^ 1], ax.nwords);
  Win wn;
  const unsigned lane = lane_id(), wib = threadIdx.x >> 5;
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  unsigned long long my_edges = 0, my_act = 0;
  uint32_t my_min = INF, my_push = 0;

  // heavy slots: static 1024-edge chunks of rows with out-degree > HEAVY_DEG.
  // This warp owns chunks gw + nw*k; its lanes test 32 of them at once (one
  // round of dependent loads instead of 32) and the warp relaxes the active ones.
  const int64_t my_chunks = ax.nhc > gw ? (ax.nhc - gw + nw - 1) / nw : 0;
  for (int64_t k0 = 0; k0 < my_chunks; k0 += 32) {
    const int64_t kc = k0 + lane;
    int32_t uc = -1;
    if (kc < my_chunks) {
      uc = ax.hc_row[gw + nw * kc];
      if (uc < row_lo || uc >= row_hi || !bit_of(bm_cur, (uint32_t)uc)) uc = -1;   // another rank's rows (dist.h)
    }
    unsigned todo = __ballot_sync(FULL, uc >= 0);
    while (todo) {
      const int l = __ffs(todo) - 1;
      todo &= todo - 1;
      const int64_t c = gw + nw * (k0 + l);
      const int32_t u = __shfl_sync(FULL, uc, l);
      uint32_t a = ax.hc_start[c];
      uint32_t b = min(a + HCHUNK, rp[u + 1]);
      const uint32_t du = ld_l2_u32(dist + u, pl);
      if (a == rp[u] && lane == 0) my_act++;
      if (lh) {   // the chunk's light / heavy part
        const uint32_t le = ax.lend[u];
        if (lh == 1) b = min(b, le);
        else a = max(a, le);
        if (a >= b) continue;
      }
      uint2 ed[SU];
      bool ok[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) {
        const uint32_t e = a + q * 32 + lane;
        ok[q] = e < b;
        ed[q] = ok[q] ? ld_edge(adj, ax, e, pf) : make_uint2(0, 0);
      }
      for (uint32_t e0 = a; e0 < b; e0 += 32 * SU) {
        // the next round's edges are loaded before this round's gathers
        uint2 en[SU];
        bool kn[SU];
#pragma unroll
        for (int q = 0; q < SU; q++) {
          const uint32_t e = e0 + 32 * SU + q * 32 + lane;
          kn[q] = e < b;
          en[q] = kn[q] ? ld_edge(adj, ax, e, pf) : make_uint2(0, 0);
        }
        uint32_t cv[SU];
#pragma unroll
        for (int q = 0; q < SU; q++) cv[q] = ok[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
        for (int q = 0; q < SU; q++)
          if (ok[q]) relax_nf(ed[q], du, cv[q], dist, bm_next, ax.far, tau, my_min, my_push, pl, wn);
#pragma unroll
        for (int q = 0; q < SU; q++) {
          ed[q] = en[q];
          ok[q] = kn[q];
        }
      }
      if (lane == 0) my_edges += b - a;
    }
  }

  // light slots: each warp compacts the frontier bits of 32 bitmap words into
  // shared memory and relaxes them 32 slots per round.  The words of a warp
  // are strided by the warp count (word = lo + gw + nw * j), so frontiers that
  // cluster in id space (e.g. after the §2 BFS renumbering) still spread over
  // all warps, while sparse random frontiers still batch up to 1024 slots.
  int32_t* sv = s_v[wib];
  // word w_base + gw + nw*jj belongs to warp gw; the frontier window only
  // narrows the jj range, so a word keeps its warp (the processing order of a
  // wavefront stays that of the full scan: a shifted assignment measured 35 %
  // more relaxations on the road grid's wide buckets)
  const int64_t w_base = row_lo >> 5;                                        // ranges are 32-aligned
  int64_t w_lo = w_base, w_hi = min((row_hi + 31) >> 5, ax.nwords);
  if (win) {
    w_lo = max(w_lo, (int64_t)st->wlo[t % 6]);
    w_hi = min(w_hi, (int64_t)st->whi[t % 6] + 1);
  }
  const int64_t my_words = w_hi > w_base + gw ? (w_hi - w_base - gw + nw - 1) / nw : 0;   // jj < my_words
  const int64_t jj0 = w_lo > w_base + gw ? (w_lo - w_base - gw + nw - 1) / nw : 0;     // first jj in the window
  // the frontier words of SCAN_B rounds are loaded together (one memory
  // latency instead of SCAN_B when the frontier is sparse, as on road grids)
  constexpr int SCAN_B = 4;
  for (int64_t jb = jj0; jb < my_words; jb += 32 * SCAN_B) {
    uint32_t wv[SCAN_B];
#pragma unroll
    for (int b = 0; b < SCAN_B; b++) {
      const int64_t jj = jb + 32 * b + lane;
      const int64_t wi = w_base + gw + nw * jj;
      uint32_t raw = 0u;
      if (jj < my_words) {
        raw = __ldcg(bm_cur + wi);
        // this warp owns word wi in every sweep: a plain read-modify-write
        if (pend_w && raw) __stcg(pend_w + wi, __ldcg(pend_w + wi) | raw);
      }
      wv[b] = raw ? (raw & ~__ldg(ax.heavy + wi)) : 0u;
    }
    uint32_t anyw = 0;
#pragma unroll
    for (int b = 0; b < SCAN_B; b++) anyw |= wv[b];
    if (!__any_sync(FULL, anyw != 0)) continue;
#pragma unroll 1
  for (int b = 0; b < SCAN_B; b++) {
    const int64_t jj = jb + 32 * b + lane;
    const int64_t wi = w_base + gw + nw * jj;
    uint32_t word = wv[b];
    const uint32_t cnt = __popc(word);
    const uint32_t incl = warp_incl_scan_u32(cnt);
    const uint32_t total = __shfl_sync(FULL, incl, 31);
    if (total == 0) continue;
    uint32_t k = incl - cnt;
    while (word) {
      const int b = __ffs(word) - 1;
      sv[k++] = (int32_t)(wi * 32 + b);
      word &= word - 1;
    }
    __syncwarp();
    for (uint32_t base = 0; base < total; base += 32) {
      const uint32_t idx = base + lane;
      const bool mine = idx < total;
      uint32_t start = 0, deg = 0, du = 0;
      if (mine) {
        const int32_t u = sv[idx];
        du = ld_l2_u32(dist + u, pl);
#if GX_SSSP_RP_EF
        start = ld_l2_u32(rp + u, pf);   // keep the L2 for the gathered dist
        uint32_t end = ld_l2_u32(rp + u + 1, pf);
#else
        start = rp[u];
        uint32_t end = rp[u + 1];
#endif
        if (lh == 1) end = ax.lend[u];
        else if (lh == 2) start = ax.lend[u];
        deg = end - start;
        my_act++;
      }
      const uint32_t dincl = warp_incl_scan_u32(deg);
      const uint32_t dexcl = dincl - deg;
      const uint32_t dtot = __shfl_sync(FULL, dincl, 31);
      // round k0: the SU edges k0 + q*32 + lane of the batch's concatenated rows
      // (binary search of the owning row over the warp's exclusive scan)
      auto fetch = [&](uint32_t k0, uint2 (&ed)[SU], uint32_t (&od)[SU], bool (&ok)[SU]) {
#pragma unroll
        for (int q = 0; q < SU; q++) {
          const uint32_t kk = k0 + q * 32 + lane;
          int j = 0;
#pragma unroll
          for (int sft = 16; sft; sft >>= 1) {
            uint32_t ex = __shfl_sync(FULL, dexcl, j + sft);
            if (ex <= kk) j += sft;
          }
          const uint32_t os = __shfl_sync(FULL, start, j);
          const uint32_t oe = __shfl_sync(FULL, dexcl, j);
          od[q] = __shfl_sync(FULL, du, j);
          ok[q] = kk < dtot;
          ed[q] = ok[q] ? ld_edge(adj, ax, os + (kk - oe), pf) : make_uint2(0, 0);
        }
      };
#if GX_SSSP_PIPE
      // software pipeline: round k0 + 32*SU's edge loads are issued before
      // round k0's dist gathers, so each lane keeps 2*SU loads in flight and
      // the edge-stream latency hides behind the gathers'
      uint2 ed[SU];
      uint32_t od[SU];
      bool ok[SU];
      if (dtot) fetch(0, ed, od, ok);
      for (uint32_t k0 = 0; k0 < dtot; k0 += 32 * SU) {
        const bool more = k0 + 32 * SU < dtot;   // warp-uniform
        uint2 en[SU];
        uint32_t on[SU];
        bool kn[SU];
        if (more) fetch(k0 + 32 * SU, en, on, kn);
        uint32_t cv[SU];
#pragma unroll
        for (int q = 0; q < SU; q++) cv[q] = ok[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
        for (int q = 0; q < SU; q++)
          if (ok[q]) relax_nf(ed[q], od[q], cv[q], dist, bm_next, ax.far, tau, my_min, my_push, pl, wn);
        if (more) {
#pragma unroll
          for (int q = 0; q < SU; q++) {
            ed[q] = en[q];
            od[q] = on[q];
            ok[q] = kn[q];
          }
        }
      }
#else
      for (uint32_t k0 = 0; k0 < dtot; k0 += 32 * SU) {
        uint2 ed[SU];
        uint32_t od[SU];
        bool ok[SU];
        fetch(k0, ed, od, ok);
        uint32_t cv[SU];
#pragma unroll
        for (int q = 0; q < SU; q++) cv[q] = ok[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
        for (int q = 0; q < SU; q++)
          if (ok[q]) relax_nf(ed[q], od[q], cv[q], dist, bm_next, ax.far, tau, my_min, my_push, pl, wn);
      }
#endif
      if (lane == 0) my_edges += dtot;
    }
    __syncwarp();
  }
  }
  flush_counters(st, t, my_edges, my_act, my_push, my_min, fdst);
  if (win) flush_windows(wn, &st->wlo[(t + 1) % 6], &st->whi[(t + 1) % 6], &st->flo[far_slot], &st->fhi[far_slot]);
}

__global__ void __launch_bounds__(256) k_sssp_lb(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj,
                                                 uint32_t* __restrict__ dist, SsspAux ax, SsspState* __restrict__ st,
                                                 int64_t row_lo, int64_t row_hi) {
  if (st->stop) return;
  const unsigned t = st->iter;
  // near-far: relaxations to dist >= tau go to the far pile
  const uint32_t tau = st->tau;
  if (blockIdx.x == 0 && threadIdx.x == 0) st->split = 0;   // the split kernel of t-1 is done
  __shared__ int32_t s_v[SB_WARPS][1024];
  sssp_lb_dev(rp, adj, dist, ax, st, row_lo, row_hi, t, tau, &st->far_min, s_v);
}

// ---------------------------------------------------------------- TPV sweep
// The paper's mapping (tpv.cu): one warp per 32-slot slice of the schedule,
// lane = slot; a lane whose slot is in the frontier walks its row in the
// SELL-32 slab (one coalesced 256-byte load per column).  The warp runs as
// long as its longest active row -- the divergence that §4 normalises.
__global__ void __launch_bounds__(256) k_sssp_tpv(const int32_t* __restrict__ lane_row, const uint32_t* __restrict__ slen,
                                                  const uint64_t* __restrict__ soff, const uint2* __restrict__ slab,
                                                  int64_t nslices, uint32_t* __restrict__ dist, SsspAux ax,
                                                  SsspState* __restrict__ st) {
  const unsigned t = st->iter;
  if (st->stop) return;
  const uint32_t* __restrict__ bm_cur = ax.bm[t % 3];
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  clear_bitmap(ax.bm[(t + 2) % 3], ax.nwords);
  const unsigned lane = lane_id();
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  unsigned long long my_edges = 0, my_act = 0;
  uint32_t my_push = 0;
  for (int64_t sl = gw; sl < nslices; sl += nw) {
    const int32_t row = lane_row[sl * 32 + lane];
    const bool act = row >= 0 && bit_of(bm_cur, (uint32_t)row);
    if (!__any_sync(FULL, act)) continue;
    my_act += act;
    const uint32_t du = act ? ld_l2_u32(dist + row, pl) : 0u;
    const uint32_t L = slen[sl];
    const uint2* p = slab + soff[sl] + lane;
    for (uint32_t j = 0; j < L; j += SU) {
      uint2 ed[SU];
      bool ok[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) {
        ed[q] = (act && j + q < L) ? ld_stream_u2(p + 32 * (j + q), pf) : make_uint2(0xFFFFFFFFu, 0u);
        ok[q] = ed[q].x != 0xFFFFFFFFu;
      }
      uint32_t cv[SU];
#pragma unroll
      for (int q = 0; q < SU; q++) cv[q] = ok[q] ? ld_l2_u32(dist + ed[q].x, pl) : 0u;
#pragma unroll
      for (int q = 0; q < SU; q++) {
        if (ok[q]) relax_red(ed[q], du, cv[q], dist, bm_next, my_push, pl);
        my_edges += ok[q];
      }
    }
  }
  flush_counters(st, t, my_edges, my_act, my_push, INF);
}

// ---------------------------------------------------------------- §3 local pass
// One CTA per subgraph tile: member distances staged in shared memory,
// relaxed t times over the tile's local edges (P@32188-32416, reading R28),
// improvements written back with atomic min and added to the next frontier.
// Touched-tile list (tlist != nullptr): the tiles with a member in the current
// or the next frontier, collected by sssp_tiles_collect_dev, so the pass costs
// O(touched tiles) instead of a scan of every tile per iteration (a road grid
// has ~4e5 tiles and ~1e4 iterations).
__device__ __forceinline__ void sssp_tiles_collect_dev(const SsspAux& ax, SsspState* __restrict__ st, unsigned t,
                                                       const int32_t* __restrict__ slot_tile,
                                                       uint32_t* __restrict__ tmark, int32_t* __restrict__ tlist) {
  const uint32_t* bm_cur = ax.bm[t % 3];
  const uint32_t* bm_next = ax.bm[(t + 1) % 3];
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < ax.nwords; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = __ldcg(bm_cur + w) | __ldcg(bm_next + w);
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      const int32_t tl = slot_tile[w * 32 + b];
      if (tl < 0) continue;
      const uint32_t bit = 1u << (tl & 31);
      if (!(atomicOr(tmark + (tl >> 5), bit) & bit)) tlist[atomicAdd(&st->tiles_n[t % 3], 1u)] = tl;
    }
  }
}
__global__ void k_sssp_tiles_collect(SsspAux ax, SsspState* __restrict__ st, const int32_t* __restrict__ slot_tile,
                                     uint32_t* __restrict__ tmark, int32_t* __restrict__ tlist) {
  if (st->stop) return;
  sssp_tiles_collect_dev(ax, st, st->iter, slot_tile, tmark, tlist);
}

// One WARP per tile (tiles hold S_max <= 256 members; the C3 road grid's
// average 3.1): the members' distances go to the warp's slice of shared
// memory, the tile's local edges ({src | dst << 8, w}) are relaxed
// warp-stride for up to t rounds (or to the local fixed point: no lane
// improved anything), improvements written back with red.min + the next
// frontier bit.  A tile's first 64 edges stay in registers across the rounds
// (2 per lane), so a small tile reads its edges from global memory once.
// No CTA barriers: warps of a CTA work on different tiles independently.
constexpr int LOCAL_MAX_MEMBERS = 256;   // u8 member indices
__device__ __forceinline__ void sssp_local_dev(const int32_t* __restrict__ tptr, const int32_t* __restrict__ tmem,
                                               const int32_t* __restrict__ teptr, const uint2* __restrict__ tedges,
                                               const int32_t* __restrict__ titers, int64_t ntiles,
                                               uint32_t* __restrict__ dist, const SsspAux& ax, SsspState* __restrict__ st,
                                               const int32_t* __restrict__ tlist, uint32_t* __restrict__ tmark,
                                               uint32_t* __restrict__ pool /* blockDim/32 x LOCAL_MAX_MEMBERS */) {
  const unsigned t = st->iter;
  if (st->stop) return;
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  const uint64_t pl = l2_evict_last();
  const uint32_t* bm_cur = ax.bm[t % 3];
  const unsigned lane = lane_id();
  uint32_t* sd = pool + (threadIdx.x >> 5) * LOCAL_MAX_MEMBERS;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t my_push = 0;
  const int64_t nwork = tlist ? (int64_t)*(volatile unsigned*)&st->tiles_n[t % 3] : ntiles;
  for (int64_t wi = gw; wi < nwork; wi += nw) {
    const int64_t tile = tlist ? tlist[wi] : wi;
    const int a = tptr[tile], nm = tptr[tile + 1] - a;
    const int ea = teptr[tile], ne = teptr[tile + 1] - ea;
    if (tlist) {
      if (lane == 0) atomicAnd(tmark + (tile >> 5), ~(1u << (tile & 31)));   // listed once per iteration
    } else {
      // only tiles touched by this iteration: a member in the frontier or improved by the sweep
      bool touched = false;
      for (int i = lane; i < nm; i += 32) {
        const uint32_t v = (uint32_t)tmem[a + i];
        touched |= (((__ldcg(bm_cur + (v >> 5)) | __ldcg(bm_next + (v >> 5))) >> (v & 31)) & 1u) != 0;
      }
      if (!__any_sync(FULL, touched)) continue;
    }
    for (int i = lane; i < nm; i += 32) sd[i] = ld_l2_u32(dist + tmem[a + i], pl);
    // the first 64 local edges in registers
    uint2 e0 = lane < ne ? tedges[ea + lane] : make_uint2(0, 0);
    uint2 e1 = lane + 32 < ne ? tedges[ea + 32 + lane] : make_uint2(0, 0);
    __syncwarp();
    const int iters = titers[tile];
    auto relax = [&](uint2 p) -> bool {
      const uint32_t du = sd[p.x & 0xff];
      if (du == INF) return false;
      const uint32_t nd = sat_add(du, p.y);
      const uint32_t dst = (p.x >> 8) & 0xff;
      if (nd < sd[dst]) {
        atomicMin(&sd[dst], nd);
        return true;
      }
      return false;
    };
    for (int r = 0; r < iters; r++) {
      bool ch = false;
      if (lane < ne) ch |= relax(e0);
      if (lane + 32 < ne) ch |= relax(e1);
      for (int i = 64 + lane; i < ne; i += 32) ch |= relax(tedges[ea + i]);
      if (!__any_sync(FULL, ch)) break;
      __syncwarp();
    }
    __syncwarp();
    for (int i = lane; i < nm; i += 32) {
      const uint32_t v = (uint32_t)tmem[a + i];
      const uint32_t nd = sd[i];
      if (nd < ld_l2_u32(dist + v, pl)) {
        red_min_l2(dist + v, nd, pl);
        red_or_l2(bm_next + (v >> 5), 1u << (v & 31), pl);
        my_push++;
      }
    }
    __syncwarp();
  }
  flush_counters(st, t, 0, 0, my_push, INF);
}

__global__ void __launch_bounds__(256) k_sssp_local(const int32_t* __restrict__ tptr, const int32_t* __restrict__ tmem,
                                                    const int32_t* __restrict__ teptr, const uint2* __restrict__ tedges,
                                                    const int32_t* __restrict__ titers, int64_t ntiles,
                                                    uint32_t* __restrict__ dist, SsspAux ax, SsspState* __restrict__ st,
                                                    const int32_t* __restrict__ tlist, uint32_t* __restrict__ tmark) {
  __shared__ uint32_t pool[(256 / 32) * LOCAL_MAX_MEMBERS];
  sssp_local_dev(tptr, tmem, teptr, tedges, titers, ntiles, dist, ax, st, tlist, tmark, pool);
}

// ---------------------------------------------------------------- §2.4 merge
// One warp per confluence group.  The owner first re-pulls its in-edges (the
// Jacobi step a merge may have undone), then all
// copies take the mean (floor of the exact 64-bit mean, INF copies excluded,
// reading R19) or the min (GX_MERGE_MIN).  Copies that decrease re-enter the
// frontier.
__device__ __forceinline__ void sssp_merge_dev(const int32_t* __restrict__ gptr, const int32_t* __restrict__ gslots,
                                               const int32_t* __restrict__ ginptr, const uint2* __restrict__ gin,
                                               int64_t ngroups, int merge_min, uint32_t* __restrict__ dist,
                                               const SsspAux& ax, SsspState* __restrict__ st) {
  const unsigned t = st->iter;
  if ((st->stop && st->stop != 4) || !st->do_merge) return;   // 4: a blocked dense iteration in progress
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  const unsigned lane = lane_id();
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t my_push = 0;
  for (int64_t gi = warp; gi < ngroups; gi += nw) {
    const int a = gptr[gi], b = gptr[gi + 1];
    const int32_t o = gslots[a];
    uint32_t best = INF;
    for (int e = ginptr[gi] + lane; e < ginptr[gi + 1]; e += 32) {
      const uint2 iv = gin[e];
      const uint32_t dp = __ldcg(dist + iv.x);
      if (dp != INF) best = min(best, sat_add(dp, iv.y));   // saturating (R51)
    }
    best = warp_min_u32(best);
    const uint32_t own = min(__ldcg(dist + o), best);
    unsigned long long sum = 0;
    unsigned cnt = 0;
    uint32_t mn = INF;
    for (int i = a + lane; i < b; i += 32) {
      const uint32_t val = (i == a) ? own : __ldcg(dist + gslots[i]);
      if (val != INF) {
        sum += val;
        cnt++;
      }
      mn = min(mn, val);
    }
    sum = warp_sum_u64(sum);
    cnt = __reduce_add_sync(FULL, cnt);
    mn = warp_min_u32(mn);
    const uint32_t mval = merge_min ? mn : (cnt ? (uint32_t)(sum / cnt) : INF);
    for (int i = a + lane; i < b; i += 32) {
      const uint32_t sl = (uint32_t)gslots[i];
      const uint32_t old = __ldcg(dist + sl);
      if (old != mval) {
        dist[sl] = mval;
        if (mval < old) {
          atomicOr(bm_next + (sl >> 5), 1u << (sl & 31));
          my_push++;
        } else {
          atomicAdd(&st->raised, 1u);
        }
      }
    }
  }
  flush_counters(st, t, 0, 0, my_push, INF);
}

__global__ void __launch_bounds__(256) k_sssp_merge(const int32_t* __restrict__ gptr, const int32_t* __restrict__ gslots,
                                                    const int32_t* __restrict__ ginptr, const uint2* __restrict__ gin,
                                                    int64_t ngroups, int merge_min, uint32_t* __restrict__ dist,
                                                    SsspAux ax, SsspState* __restrict__ st) {
  sssp_merge_dev(gptr, gslots, ginptr, gin, ngroups, merge_min, dist, ax, st);
}

// merge cadence c != 1 (P@28188: "after a certain number of iterations or at
// the end of the overall computation"): decided once per iteration,
// before the merge kernel, from the sweep's counters.  c > 1: merge after
// every c-th iteration and whenever the sweep alone reached its fixed point
// (so the run still ends at a merged fixed point); c = 0: only then, and that
// merge ends the run (copies keep the mean; what it pushes is not relaxed).
__device__ __forceinline__ void sssp_merge_decide_dev(SsspState* __restrict__ st) {
  if (st->stop) return;
  const unsigned t = st->iter, c = st->merge_every;
  const bool fixed = st->pushed[t % 3] == 0 && st->far_min == INF;
  st->do_merge = ((c > 1 && ((t + 1) % c == 0 || fixed)) || (c == 0 && fixed)) ? 1u : 0u;
  st->final_merge = (c == 0 && fixed) ? 1u : 0u;
}
__global__ void k_sssp_merge_decide(SsspState* __restrict__ st) { sssp_merge_decide_dev(st); }

// end of iteration t: no bit was set in the next frontier and the far pile is
// empty => converged (every decreased slot has been relaxed)
__device__ __forceinline__ void sssp_advance_dev(SsspState* __restrict__ st, int max_iters) {
  if (st->stop) return;
  const unsigned t = st->iter;
  if (st->final_merge) {
    st->act_total += st->active[t % 3];
    st->stop = 1;
    st->iter = t + 1;
    return;
  }
  st->act_total += st->active[t % 3];
  st->active[(t + 2) % 3] = 0;
  st->pushed[(t + 2) % 3] = 0;
  st->tiles_n[(t + 2) % 3] = 0;
  if (st->pushed[t % 3] == 0) {  // the next frontier is empty
    if (st->far_min == INF) {    // ... and so is the far pile
      st->stop = 1;
      st->iter = t + 1;
      return;
    }
    // the bucket drained: raise the threshold past the nearest far slot and
    // let k_sssp_split move the far slots below it into the next frontier
    const unsigned long long nt = (unsigned long long)st->far_min + st->delta;
    st->tau = nt >= INF ? INF : (unsigned)nt;
    st->far_min = INF;
    st->split = 1;
  }
  st->iter = t + 1;
  if ((int)(t + 1) >= max_iters) st->stop = 2;
}
__global__ void k_sssp_advance(SsspState* __restrict__ st, int max_iters) { sssp_advance_dev(st, max_iters); }

// near-far refill (after k_sssp_advance raised tau): far slots of this rank's
// range with dist < tau join the frontier of the new iteration; the rest stay
// and re-establish far_min
// t = the iteration the refilled frontier belongs to; remaining far minimum -> fdst
__device__ __forceinline__ void sssp_split_dev(const uint32_t* __restrict__ dist, const SsspAux& ax,
                                               SsspState* __restrict__ st, int64_t lo, int64_t hi, const unsigned t,
                                               const uint32_t tau, uint32_t* fdst,
                                               const uint32_t* __restrict__ rp = nullptr, const bool win = false,
                                               const unsigned fslot = 0, const uint32_t tau_prev = 0) {
  // win: the far pile's bits lie in words [flo[fslot], fhi[fslot]]; the moved
  // bits' words widen bm[t%3]'s window, the kept bits' words form the far
  // window of the next epoch (slot fslot ^ 1, empty before)
  uint32_t* bm_cur = ax.bm[t % 3];
  uint32_t my_min = INF;
  unsigned long long my_deg = 0;   // the moved slots (dense-iteration test, adaptive window)
  Win wn;
  if (!ax.far) {
    // far pile by scan (ax.far null: no far bitmap, the persistent loop on
    // graphs without merges / tiles / windows): the far pile is exactly the
    // rows with tau_prev <= dist < INF.  A row is only ever processed in a
    // near frontier at a value below that frontier's tau <= tau_prev, and dist
    // only decreases, so a row at >= tau_prev was never processed at its value;
    // a row below tau_prev was processed at its value or still waits in the
    // near frontier (early refill).  One coalesced read of dist per refill
    // instead of a red.or per far push (and no stale far bits re-activated)
    const int64_t gwp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwp = ((int64_t)gridDim.x * blockDim.x) >> 5;
    // 128 slots (4 bitmap words) per warp load: lane l holds slots 4l..4l+3
    // (one uint4), its 4-bit move mask is OR-reduced over the 8 lanes of a
    // word; FS_U chunks per warp loaded together.  lo == 0 (persistent loop).
    const unsigned lane = lane_id();
    const int64_t c_end = (hi + 127) >> 7;
    constexpr int FS_U = 4;
    for (int64_t cb = gwp; cb < c_end; cb += nwp * FS_U) {
      uint4 q[FS_U];
#pragma unroll
      for (int k = 0; k < FS_U; k++) {
        const int64_t ch = cb + k * nwp;
        const int64_t v = ch * 128 + 4 * lane;
        if (ch < c_end && v + 3 < hi) {
          q[k] = __ldcg(reinterpret_cast<const uint4*>(dist + v));
        } else {
          const bool in = ch < c_end;
          q[k].x = in && v < hi ? __ldcg(dist + v) : INF;
          q[k].y = in && v + 1 < hi ? __ldcg(dist + v + 1) : INF;
          q[k].z = in && v + 2 < hi ? __ldcg(dist + v + 2) : INF;
          q[k].w = INF;
        }
      }
#pragma unroll
      for (int k = 0; k < FS_U; k++) {
        const uint32_t dd[4] = {q[k].x, q[k].y, q[k].z, q[k].w};
        unsigned nib = 0;
#pragma unroll
        for (int c = 0; c < 4; c++) {
          if (dd[c] >= tau_prev && dd[c] < tau) nib |= 1u << c;
          if (dd[c] >= tau && dd[c] != INF) my_min = min(my_min, dd[c]);
        }
        unsigned x = nib << (4 * (lane & 7));
        x |= __shfl_xor_sync(FULL, x, 1);
        x |= __shfl_xor_sync(FULL, x, 2);
        x |= __shfl_xor_sync(FULL, x, 4);
        if ((lane & 7) == 0 && x) {
          atomicOr(bm_cur + (cb + k * nwp) * 4 + (lane >> 3), x);   // RED: the word may hold near pushes
          my_deg += __popc(x);
        }
      }
    }
  }
  int64_t w_lo = lo >> 5, w_hi = ax.far ? min((hi + 31) >> 5, ax.nwords) : w_lo;
  if (win) {
    w_lo = max(w_lo, (int64_t)st->flo[fslot]);
    w_hi = min(w_hi, (int64_t)st->fhi[fslot] + 1);
  }
  for (int64_t w = w_lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < w_hi; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = ax.far[w];
    if (!bits) continue;
    uint32_t move = 0, keep = bits;
    while (bits) {
      const int b = __ffs(bits) - 1;
      bits &= bits - 1;
      const uint32_t d = dist[w * 32 + b];
      if (d < tau) {
        move |= 1u << b;
      } else {
        my_min = min(my_min, d);
      }
    }
    keep &= ~move;
    ax.far[w] = keep;
    if (move) {
      bm_cur[w] |= move;
      wn.nlo = min(wn.nlo, (uint32_t)w);
      wn.nhi = max(wn.nhi, (uint32_t)w);
    }
    if (keep) {
      wn.flo = min(wn.flo, (uint32_t)w);
      wn.fhi = max(wn.fhi, (uint32_t)w);
    }
    my_deg += __popc(move);
  }
  (void)rp;
  my_deg = warp_sum_u64(my_deg);
  if (lane_id() == 0 && my_deg) atomicAdd(&st->refill_deg[t % 3], my_deg);
  flush_counters(st, 0, 0, 0, 0, my_min, fdst);
  if (win) flush_windows(wn, &st->wlo[t % 6], &st->whi[t % 6], &st->flo[fslot ^ 1u], &st->fhi[fslot ^ 1u]);
}
__global__ void k_sssp_split(const uint32_t* __restrict__ dist, SsspAux ax, SsspState* __restrict__ st, int64_t lo,
                             int64_t hi) {
  if (st->stop || !st->split) return;
  sssp_split_dev(dist, ax, st, lo, hi, st->iter, st->tau, &st->far_min);
}

// ---------------------------------------------------------------- block-local mode
// For graphs whose edges mostly stay inside contiguous id blocks (road grids
// in their natural row-major order: ~10^4 iterations of a few thousand slots
// each), CTA b owns rows [b*B, (b+1)*B).  In each global iteration it relaxes
// the frontier slots of its block and keeps propagating improvements of its
// OWN rows through a shared-memory work queue for up to BLK_ROUNDS local
// rounds, so a wave crosses many hops per grid barrier (the paper's §3 idea
// -- iterate a subgraph in shared memory, P@32188 -- applied exactly, to the
// id blocks, without added edges).  Improvements of other blocks' rows (and
// queue overflow) go to the global next frontier as usual.  Any relaxation
// order reaches the same fixed point (monotone min; Theorem E1's argument).
constexpr int BLK_MAX = 65536;   // rows per block (in-queue bitmap = 8 KB of shared memory)
constexpr int BLK_Q = 2048;      // entries per local queue buffer (two buffers)
constexpr int BLK_ROUNDS = 256;  // local rounds per global iteration

__device__ __forceinline__ void sssp_block_dev(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj,
                                               uint32_t* __restrict__ dist, const SsspAux& ax,
                                               SsspState* __restrict__ st, int64_t n_slots, int64_t B,
                                               const unsigned t, const uint32_t tau, uint32_t* fdst,
                                               uint8_t* pool) {
  // shared memory (aliases the LB sweep's compaction buffer): two queues,
  // the in-queue bitmap of the block, two counters
  int32_t (*q)[BLK_Q] = reinterpret_cast<int32_t (*)[BLK_Q]>(pool);
  uint32_t* inq = reinterpret_cast<uint32_t*>(pool + 2 * BLK_Q * 4);
  int* s_cnt = reinterpret_cast<int*>(pool + 2 * BLK_Q * 4 + BLK_MAX / 8);
  const uint32_t* __restrict__ bm_cur = ax.bm[t % 3];
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  clear_bitmap(ax.bm[(t + 2) % 3], ax.nwords);
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const int64_t lo = (int64_t)blockIdx.x * B, hi = min(n_slots, lo + B);
  unsigned long long my_edges = 0, my_act = 0;
  uint32_t my_min = INF, my_push = 0;
  if (lo < hi) {
    const int nw_blk = (int)((hi - lo + 31) >> 5);
    for (int i = threadIdx.x; i < nw_blk; i += blockDim.x) inq[i] = 0;
    if (threadIdx.x < 2) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    int cur = 0;
    // relax the out-edges of u; own-block improvements below tau are queued
    auto relax_vertex = [&](int32_t u) {
      const uint32_t du = ld_l2_u32(dist + u, pl);
      const uint32_t a = rp[u], b = rp[u + 1];
      my_act++;
      my_edges += b - a;
      for (uint32_t e = a; e < b; e++) {
        const uint2 ed = ld_edge(adj, ax, e, pf);
        const uint32_t nd = sat_add(du, ed.y);
        const uint32_t cv = ld_l2_u32(dist + ed.x, pl);
        if (nd >= cv) continue;
        const int64_t v = ed.x;
        if (v >= lo && v < hi && nd < tau) {
          const uint32_t old = atom_min_l2(dist + v, nd, pl);
          if (nd < old) {
            const uint32_t bit = 1u << ((v - lo) & 31);
            if (!(atomicOr(&inq[(v - lo) >> 5], bit) & bit)) {
              const int k = atomicAdd(&s_cnt[cur ^ 1], 1);
              if (k < BLK_Q) {
                q[cur ^ 1][k] = (int32_t)v;
              } else {   // queue full: next global iteration
                red_or_l2(bm_next + (v >> 5), 1u << (v & 31), pl);
                my_push++;
              }
            }
          }
        } else {
          Win wn_unused;
          relax_nf(ed, du, cv, dist, bm_next, ax.far, tau, my_min, my_push, pl, wn_unused);
        }
      }
    };
    // the global frontier's slots in this block (a thread per bitmap word);
    // pushes of this pass land in q[1]
    cur = 0;
    for (int64_t w = (lo >> 5) + threadIdx.x; w < ((hi + 31) >> 5); w += blockDim.x) {
      uint32_t bits = __ldcg(bm_cur + w);
      while (bits) {
        const int b = __ffs(bits) - 1;
        bits &= bits - 1;
        relax_vertex((int32_t)(w * 32 + b));
      }
    }
    __syncthreads();
    cur = 1;
    for (int r = 0; r < BLK_ROUNDS; r++) {
      const int n = min(s_cnt[cur], BLK_Q);
      if (n == 0) break;                       // uniform: read after a barrier
      if (threadIdx.x == 0) s_cnt[cur ^ 1] = 0;
      __syncthreads();
      for (int i = threadIdx.x; i < n; i += blockDim.x) {
        const int32_t u = q[cur][i];
        atomicAnd(&inq[(u - lo) >> 5], ~(1u << ((u - lo) & 31)));
        relax_vertex(u);
      }
      __syncthreads();
      cur ^= 1;
    }
    // rounds exhausted: what is still queued joins the global next frontier
    const int n = min(s_cnt[cur], BLK_Q);
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      const int32_t u = q[cur][i];
      red_or_l2(bm_next + (u >> 5), 1u << (u & 31), pl);
      my_push++;
    }
  }
  flush_counters(st, t, my_edges, my_act, my_push, my_min, fdst);
}

__global__ void k_block_locality(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj, int64_t n, int64_t B,
                                 unsigned long long* __restrict__ out) {
  unsigned long long loc = 0;
  uint32_t mx = 0;
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t a = rp[u], b = rp[u + 1];
    mx = max(mx, b - a);
    for (uint32_t e = a; e < b; e++) loc += (adj[e].x / B) == (u / B);
  }
  loc = warp_sum_u64(loc);
  mx = warp_max_u32(mx);
  if (lane_id() == 0) {
    atomicAdd(out, loc);
    atomicMax(out + 1, (unsigned long long)mx);
  }
}

// ---------------------------------------------------------------- persistent loop
// The whole fixed-point loop of the LB mapping in ONE cooperative launch:
// every phase of an iteration (sweep, §3 local pass, §2.4 merge, advance,
// near-far refill) runs on the resident grid, separated by grid-wide
// barriers, instead of 3-5 kernel launches per iteration.  What it removes is
// the per-iteration fixed cost (launch gaps, kernel prologues), which is what
// bounds high-diameter graphs: a road grid needs ~10^4 iterations whose
// frontiers are a few thousand slots.  grid.sync() is a gpu-scope
// release/acquire (MEMBAR.GPU + CCTL.IVALL in SASS), so every phase sees the
// previous phase's writes; the loop state is read only after a barrier.
struct SsspLoop {
  const uint32_t* rp;
  const uint2* adj;
  uint32_t* dist;
  SsspAux ax{};
  SsspState* st;
  int64_t n_slots;
  const int32_t *tptr, *tmem, *teptr, *titers;
  const uint2* tedges;
  int64_t ntiles;
  const int32_t *gptr, *gslots, *ginptr;
  const uint2* gin;
  int64_t ngroups;
  int merge_min, cadence, max_iters;
  unsigned early;       // refill the next bucket once the near frontier's pushes are <= early (0: only when empty)
  unsigned long long small_refill;   // a refill moving fewer slots doubles the next window (up to wmul_cap)
  unsigned wmul_cap;
  int64_t block_rows;   // > 0: block-local mode with this many rows per CTA
  const int32_t* slot_tile;
  uint32_t* tmark;
  int32_t* tlist;
  unsigned long long* trace;   // GX_SSSP_PTRACE: per iteration {globaltimer ns, edges so far, active, tau}
  int trace_cap;
  unsigned long long dense_edges;   // > 0: a refill that moves >= this many slots exits for the blocked
                                    // dense relaxation (stop = 4); 0: never
};

constexpr int PERSIST_POOL = SB_WARPS * 1024 * 4;   // 32 KB at 256 threads: LB compaction buffer / block-mode queues
static_assert(2 * BLK_Q * 4 + BLK_MAX / 8 + 16 <= PERSIST_POOL, "block-mode buffers must fit the pool");
static_assert((PERSIST_TPB / 32) * LOCAL_MAX_MEMBERS * 4 <= PERSIST_POOL, "local-pass slices must fit the pool");

#ifndef GX_SSSP_MINB
#define GX_SSSP_MINB (1024 / GX_SSSP_TPB)
#endif
__global__ void __launch_bounds__(PERSIST_TPB, GX_SSSP_MINB) k_sssp_persist(SsspLoop a) {
  __shared__ __align__(16) uint8_t pool[PERSIST_POOL];
  cg::grid_group grid = cg::this_grid();
  const bool lead = blockIdx.x == 0 && threadIdx.x == 0;
  SsspState* st = a.st;
  // Loop control is replicated: after the sweep's barrier every thread reads
  // the same counters and takes the same decision (stop / refill / new tau),
  // so no barrier is needed between the decision and the next sweep.  The
  // lead thread mirrors the state into *st for the host and clears the
  // counter slots of iteration t+2 (last read at the decision of t-1, which
  // every CTA has passed).  far3[t%3] collects the far pile's minimum pushed
  // in iteration t; rf is the running minimum since the last refill.
  unsigned t = st->iter;
  uint32_t tau = st->tau, rf = st->far_min;   // a relaunch after a dense iteration continues its state
  const uint32_t delta = st->delta;
  // adaptive window: the tail buckets of a power-law graph hold few slots but
  // each refill scans the whole far pile (~1M slots on RMAT-24) -- a refill
  // that moves fewer than small_refill slots doubles the next window
  uint32_t wmul = st->wmul ? st->wmul : 1u;
  auto adapt = [&](unsigned tt) {
    const unsigned long long moved = *(volatile unsigned long long*)&st->refill_deg[tt % 3];
    wmul = moved < a.small_refill ? min(wmul * 2u, a.wmul_cap) : 1u;
    if (lead) st->wmul = wmul;
  };
  // frontier windows: the far pile's window slot is the refill epoch's parity;
  // a refill reads slot e&1 and builds slot (e+1)&1, which the lead emptied
  // after the previous refill (replicated like tau)
  const bool win = st->win_on != 0;
  unsigned epoch = st->epoch;
  auto refill = [&](unsigned tt, uint32_t tau_prev) {
    sssp_split_dev(a.dist, a.ax, st, 0, a.n_slots, tt, tau, &st->far3[tt % 3], a.dense_edges ? a.rp : nullptr, win,
                   epoch & 1u, tau_prev);
    grid.sync();
    if (lead) {
      st->flo[epoch & 1u] = 0xFFFFFFFFu;   // read by this refill only; the next refill builds it
      st->fhi[epoch & 1u] = 0u;
      st->epoch = epoch + 1;
    }
    epoch++;
  };
  // the relaunch's pending near-far refill (decided after the dense iteration)
  if (*(volatile unsigned*)&st->split) {
    refill(t, st->tau_prev);
    if (lead) st->split = 0;
    adapt(t);
    if (a.dense_edges && *(volatile unsigned long long*)&st->refill_deg[t % 3] >= a.dense_edges) {
      if (lead) st->stop = 4;
      return;
    }
  }
  // light / heavy split (ax.lend set; no tiles, merges or block mode): pend_n =
  // frontier entries since the last heavy pass, hv = this iteration is one
  const bool lh = a.ax.lend != nullptr;
  unsigned pend_n = 0;
  int pp = 0;
  bool hv = false;
  for (;;) {
    if (a.block_rows > 0)
      sssp_block_dev(a.rp, a.adj, a.dist, a.ax, st, a.n_slots, a.block_rows, t, tau, &st->far3[t % 3], pool);
    else
      sssp_lb_dev(a.rp, a.adj, a.dist, a.ax, st, 0, a.n_slots, t, tau, &st->far3[t % 3],
                  reinterpret_cast<int32_t (*)[1024]>(pool), lh ? (hv ? 2 : 1) : 0, pp, epoch & 1u, win);
    grid.sync();
    if (a.ntiles) {
      sssp_tiles_collect_dev(a.ax, st, t, a.slot_tile, a.tmark, a.tlist);
      grid.sync();
      sssp_local_dev(a.tptr, a.tmem, a.teptr, a.tedges, a.titers, a.ntiles, a.dist, a.ax, st, a.tlist, a.tmark,
                     reinterpret_cast<uint32_t*>(pool));
      grid.sync();
    }
    bool final_merge = false;
    if (a.ngroups) {
      bool doit = true;
      if (a.cadence) {   // cadence N2, same rule as k_sssp_merge_decide
        const unsigned c = st->merge_every;
        const bool fixed = *(volatile unsigned*)&st->pushed[t % 3] == 0 &&
                           min(rf, *(volatile unsigned*)&st->far3[t % 3]) == INF;
        doit = (c > 1 && ((t + 1) % c == 0 || fixed)) || (c == 0 && fixed);
        final_merge = c == 0 && fixed;
        if (lead) {
          st->do_merge = doit ? 1u : 0u;
          st->final_merge = final_merge ? 1u : 0u;
        }
        grid.sync();
      }
      if (doit) {
        sssp_merge_dev(a.gptr, a.gslots, a.ginptr, a.gin, a.ngroups, a.merge_min, a.dist, a.ax, st);
        grid.sync();
      }
    }
    // ---- decision (every thread, identical inputs)
    const uint32_t tau_b = tau;   // the bucket bound the refill's far-by-scan starts from
    const unsigned pushed = *(volatile unsigned*)&st->pushed[t % 3];
    const uint32_t fm = min(rf, *(volatile unsigned*)&st->far3[t % 3]);
    unsigned stop = 0;
    bool split = false;
    if (lh) {
      if (hv) {
        pend_n = 0;
        pp ^= 1;
      } else {
        pend_n += *(volatile unsigned*)&st->active[t % 3];
      }
    }
    hv = false;
    if (final_merge) {
      stop = 1;
    } else if (pushed == 0 && pend_n > 0) {
      hv = true;   // the bucket drained: relax the heavy edges of its slots
      rf = fm;
    } else if (pushed <= a.early && fm != INF && !lh) {
      // the bucket drained -- or its tail is down to a few slots (pushed <=
      // early): raise tau past the nearest far slot; the refill joins the tail
      // in the next frontier (any relaxation order reaches the same fixed
      // point, Theorem E1), instead of one ~10 us iteration per tail hop
      const unsigned long long nt = (unsigned long long)fm + (unsigned long long)delta * wmul;
      tau = nt >= INF ? INF : (unsigned)nt;
      rf = INF;
      split = true;
    } else if (pushed == 0) {
      if (fm == INF) {
        stop = 1;
      } else {   // the bucket drained: raise tau past the nearest far slot
        const unsigned long long nt = (unsigned long long)fm + (unsigned long long)delta * wmul;
        tau = nt >= INF ? INF : (unsigned)nt;
        rf = INF;
        split = true;
      }
    } else {
      rf = fm;
    }
    if (!stop && (int)(t + 1) >= a.max_iters) stop = 2;
    if (lead && a.trace && (int)t < a.trace_cap) {
      unsigned long long ns;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ns));
      a.trace[4 * t] = ns;
      a.trace[4 * t + 1] = *(volatile unsigned long long*)&st->edges;
      a.trace[4 * t + 2] = *(volatile unsigned*)&st->active[t % 3];
      a.trace[4 * t + 3] = tau;
    }
    if (lead) {
      st->act_total += st->active[t % 3];
      st->active[(t + 2) % 3] = 0;
      st->pushed[(t + 2) % 3] = 0;
      st->far3[(t + 2) % 3] = INF;
      st->tiles_n[(t + 2) % 3] = 0;
      st->refill_deg[(t + 2) % 3] = 0;
      st->wlo[(t + 5) % 6] = 0xFFFFFFFFu;   // frontier t-1 (bm[(t+2)%3]) was cleared by this sweep
      st->whi[(t + 5) % 6] = 0u;
      st->iter = t + 1;
      st->tau = tau;
      st->far_min = rf;
      st->stop = stop;
    }
    if (stop) break;
    t++;
    if (split) {   // near-far refill of iteration t's frontier
      refill(t, tau_b);
      adapt(t);
      // a refill that carries most of the graph's edges: hand iteration t to the
      // blocked dense relaxation (k_sssp_pb_*), which streams every edge once
      // instead of gathering dist at random for each of them
      if (a.dense_edges && *(volatile unsigned long long*)&st->refill_deg[t % 3] >= a.dense_edges) {
        if (lead) st->stop = 4;
        break;
      }
    }
  }
}

// ---------------------------------------------------------------- blocked dense relaxation
// A near-far refill that activates slots carrying most of the graph's edges
// (RMAT-24, bucket [25, 50): 8.5M slots, 205M of 268M edges) is one sparse
// matrix-vector product in the (min, +) semiring.  The LB sweep pays a random
// dist gather (one L1TEX wavefront, often across the die boundary) per edge;
// here the iteration runs over the propagation-blocked layout of the PageRank
// pull (PbLayout: edges grouped in (sink bin, source block) segments with
// 16-bit local indices) and never touches memory at random:
//   (A) k_sssp_pb_scatter: per source block, the frontier slots' distances in
//       shared memory; every edge's candidate dist[u] + w (INF for a source
//       outside the frontier) streamed to val[] (2 + 1 bytes read, 4 written)
//   (B) k_sssp_pb_gather: per sink bin, the rows' distances in shared memory,
//       the bin's candidates streamed (4 + 2 bytes) and tested against them;
//       an improving one issues a shared atomicMin (ATOMS.MIN); then the rows
//       that improved update dist and join the next frontier / far pile with
//       word-level ballots (a bin's rows are whole bitmap words)
// val[] is the PageRank layout's term array (reinterpreted as u32; PageRank
// rewrites it at the start of each run).  Same fixed point (any relaxation
// order, Theorem E1): the iteration relaxes every frontier edge exactly once.
constexpr int SPB_THREADS = 1024;
#ifndef GX_SPB_GDEPTH
#define GX_SPB_GDEPTH 4
#endif
#ifndef GX_SPB_SEGU
#define GX_SPB_SEGU 4
#endif
#ifndef GX_SPB_TEST
#define GX_SPB_TEST 1   // gather: test a candidate against the row before the atomic
#endif
constexpr int SPB_GDEPTH = GX_SPB_GDEPTH;   // gather: steps of 4 candidates per thread in flight
struct SsspPb {
  const uint32_t* q;
  const uint16_t* src_loc;
  const uint16_t* dst_loc;
  const uint16_t* w16;
  uint32_t* val;
  int64_t nb;
};

__global__ void __launch_bounds__(SPB_THREADS, 1) k_sssp_pb_scatter(SsspPb p, const uint32_t* __restrict__ dist,
                                                                    SsspAux ax, SsspState* __restrict__ st,
                                                                    int64_t n_slots) {
  extern __shared__ __align__(16) uint32_t s_d[];   // PB_R + 8: frontier distances, INF elsewhere and for padding
  if (st->stop != 4) return;
  const unsigned t = st->iter;
  const uint32_t* __restrict__ bm_cur = ax.bm[t % 3];
  const uint64_t pf = l2_evict_first();
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = SPB_THREADS / 32;
  const int64_t nb = p.nb;
  if (threadIdx.x < 8) s_d[PB_R + threadIdx.x] = INF;
  for (int64_t b = blockIdx.x; b < nb; b += gridDim.x) {
    const int64_t base = b * PB_R;
    for (int i = threadIdx.x; i < PB_R; i += SPB_THREADS) {
      const int64_t v = base + i;
      uint32_t dv = INF;
      if (v < n_slots && ((__ldcg(bm_cur + (v >> 5)) >> (v & 31)) & 1u)) dv = __ldcg(dist + v);
      s_d[i] = dv;
    }
    __syncthreads();
    const uint32_t* r0 = p.q + b * nb;   // block b's segments [r0[j], r1[j])
    const uint32_t* r1 = r0 + nb;
    // 8 entries per lane per step (16 B of source indices, 8 B of weights);
    // SPB_SEGU segments' first steps are loaded together (memory-level
    // parallelism), then each segment's remaining steps
    auto put8 = [&](uint32_t e, uint4 sx, uint4 wx) {
      const uint32_t sr[8] = {sx.x & 0xffffu, sx.x >> 16, sx.y & 0xffffu, sx.y >> 16,
                              sx.z & 0xffffu, sx.z >> 16, sx.w & 0xffffu, sx.w >> 16};
      uint32_t c[8];
#pragma unroll
      for (int i = 0; i < 8; i++) {
        const uint32_t du = s_d[sr[i]];
        const uint32_t ww = i < 2 ? wx.x : i < 4 ? wx.y : i < 6 ? wx.z : wx.w;
        const uint32_t w = (ww >> (16 * (i & 1))) & 0xffffu;
        c[i] = du == INF ? INF : sat_add(du, w);
      }
      __stcg(reinterpret_cast<uint4*>(p.val + e), make_uint4(c[0], c[1], c[2], c[3]));
      __stcg(reinterpret_cast<uint4*>(p.val + e) + 1, make_uint4(c[4], c[5], c[6], c[7]));
    };
    constexpr int SPB_SEGU = GX_SPB_SEGU;   // scatter: segments' first steps in flight per warp
    for (int64_t j0 = (int64_t)warp * 32; j0 < nb; j0 += 32 * NW) {
      const int64_t j = j0 + lane;
      const uint32_t lo = j < nb ? __ldg(r0 + j) : 0u, hi = j < nb ? __ldg(r1 + j) : 0u;
      const int kn = (int)min((int64_t)32, nb - j0);
      for (int k = 0; k < kn; k += SPB_SEGU) {
        uint32_t ee[SPB_SEGU], hh[SPB_SEGU];
        uint4 sx[SPB_SEGU];
        uint4 wx[SPB_SEGU];
#pragma unroll
        for (int u = 0; u < SPB_SEGU; u++) {
          ee[u] = __shfl_sync(FULL, lo, (k + u) & 31) + 8u * lane;
          hh[u] = k + u < kn ? __shfl_sync(FULL, hi, (k + u) & 31) : 0u;
          if (ee[u] < hh[u]) {
            sx[u] = ld_stream_v4(reinterpret_cast<const uint32_t*>(p.src_loc + ee[u]), pf);
            wx[u] = ld_stream_v4(reinterpret_cast<const uint32_t*>(p.w16 + ee[u]), pf);
          }
        }
#pragma unroll
        for (int u = 0; u < SPB_SEGU; u++) {
          if (ee[u] < hh[u]) put8(ee[u], sx[u], wx[u]);
          for (uint32_t e = ee[u] + 256u; e < hh[u]; e += 256u)
            put8(e, ld_stream_v4(reinterpret_cast<const uint32_t*>(p.src_loc + e), pf),
                 ld_stream_v4(reinterpret_cast<const uint32_t*>(p.w16 + e), pf));
        }
      }
    }
    __syncthreads();
  }
}

__global__ void __launch_bounds__(SPB_THREADS, 1) k_sssp_pb_gather(SsspPb p, uint32_t* __restrict__ dist, SsspAux ax,
                                                                   SsspState* __restrict__ st, int64_t n_slots) {
  extern __shared__ __align__(16) uint32_t acc[];   // PB_R row minima
  __shared__ int s_bin;
  if (st->stop != 4) return;
  const unsigned t = st->iter;
  const uint32_t tau = st->tau;
  const uint32_t* __restrict__ bm_cur = ax.bm[t % 3];
  uint32_t* bm_next = ax.bm[(t + 1) % 3];
  clear_bitmap(ax.bm[(t + 2) % 3], ax.nwords);
  const uint64_t pf = l2_evict_first();
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = SPB_THREADS / 32;
  const int64_t nb = p.nb;
  const uint32_t* qend = p.q + nb * nb;
  unsigned long long my_act = 0;
  uint32_t my_push = 0, my_min = INF;
  for (;;) {
    if (threadIdx.x == 0) s_bin = (int)atomicAdd(&st->dense_bin, 1u);
    __syncthreads();
    const int64_t b = s_bin;
    if (b >= nb) break;
    // the accumulator starts at the rows' current distances: a candidate is
    // tested against it first and only an improvement issues the atomic (most
    // candidates of a refill land on rows already closer, RMAT's hubs above all)
    {
      const int64_t base0 = b * PB_R;
      for (int i = threadIdx.x; i < PB_R; i += SPB_THREADS)
        acc[i] = base0 + i < n_slots ? __ldcg(dist + base0 + i) : INF;
    }
    __syncthreads();
    const uint32_t E0 = __ldg(p.q + b), E1 = __ldg(qend + b);   // multiples of 8
    // the bin's candidates: 4 per thread per step, SPB_GDEPTH steps in flight;
    // a candidate is tested against the row's current value first
    for (uint32_t e = E0 + 4u * threadIdx.x; e < E1; e += (uint32_t)SPB_GDEPTH * 4u * SPB_THREADS) {
      uint4 v[SPB_GDEPTH];
      uint2 dd[SPB_GDEPTH];
#pragma unroll
      for (int q = 0; q < SPB_GDEPTH; q++) {
        const uint32_t eq = e + (uint32_t)q * 4u * SPB_THREADS;
        v[q] = make_uint4(INF, INF, INF, INF);
        dd[q] = make_uint2(0, 0);
        if (eq < E1) {
          v[q] = ld_stream_v4(p.val + eq, pf);
          dd[q] = *reinterpret_cast<const uint2*>(p.dst_loc + eq);
        }
      }
#pragma unroll
      for (int q = 0; q < SPB_GDEPTH; q++) {
        const uint32_t vv[4] = {v[q].x, v[q].y, v[q].z, v[q].w};
        const uint32_t di[4] = {dd[q].x & 0xffffu, dd[q].x >> 16, dd[q].y & 0xffffu, dd[q].y >> 16};
#pragma unroll
        for (int i = 0; i < 4; i++)
          if (GX_SPB_TEST ? vv[i] < acc[di[i]] : vv[i] != INF) atomicMin(&acc[di[i]], vv[i]);
      }
    }
    __syncthreads();
    // the bin's rows: warp per 32 rows = one bitmap word
    const int64_t base = b * PB_R;
    const int nrows = (int)min((int64_t)PB_R, n_slots - base);
    for (int i0 = warp * 32; i0 < nrows; i0 += NW * 32) {
      const int i = i0 + lane;
      const int64_t v = base + i;
      const uint32_t nd = i < nrows ? acc[i] : INF;
      bool better = false;
      if (nd != INF) {
        const uint32_t old = __ldcg(dist + v);
        better = nd < old;
        if (better) __stcg(dist + v, nd);
      }
      const unsigned bn = __ballot_sync(FULL, better && nd < tau);
      const unsigned bf = __ballot_sync(FULL, better && nd >= tau);
      if (better && nd >= tau) my_min = min(my_min, nd);
      if (lane == 0) {
        const int64_t w = v >> 5;
        my_act += __popc(__ldcg(bm_cur + w));
        if (bn) bm_next[w] |= bn;
        if (bf && ax.far) ax.far[w] |= bf;
        my_push += __popc(bn);
      }
    }
    __syncthreads();
  }
  flush_counters(st, t, 0, my_act, my_push, my_min, &st->far3[t % 3]);
}

// the loop decision after a dense iteration t: the persistent loop's rule
// (no merges, tiles or light/heavy split in dense mode), then iteration t+1
// resumes in k_sssp_persist (a pending refill runs first there)
__global__ void k_sssp_dense_decide(SsspState* __restrict__ st, int64_t m_slots, unsigned early, int max_iters,
                                    int64_t nwords) {
  if (st->stop != 4) return;
  const unsigned t = st->iter;
  const unsigned pushed = st->pushed[t % 3];
  const uint32_t fm = min(st->far_min, st->far3[t % 3]);
  uint32_t tau = st->tau, rf = fm;
  st->tau_prev = tau;
  unsigned stop = 0, split = 0;
  if ((pushed <= early || pushed == 0) && fm != INF) {
    const unsigned long long nt = (unsigned long long)fm + (unsigned long long)st->delta * (st->wmul ? st->wmul : 1u);
    tau = nt >= INF ? INF : (unsigned)nt;
    rf = INF;
    split = 1;
  } else if (pushed == 0) {
    stop = 1;
  }
  if (!stop && (int)(t + 1) >= max_iters) stop = 2;
  st->edges += (unsigned long long)m_slots;   // every edge was scanned
  st->act_total += st->active[t % 3];
  st->active[(t + 2) % 3] = 0;
  st->pushed[(t + 2) % 3] = 0;
  st->far3[(t + 2) % 3] = INF;
  st->tiles_n[(t + 2) % 3] = 0;
  st->refill_deg[(t + 2) % 3] = 0;
  if (st->win_on) {   // the gather set bits anywhere: full windows; bm[(t+2)%3] was cleared whole
    const unsigned last = nwords > 0 ? (unsigned)(nwords - 1) : 0u;
    st->wlo[(t + 1) % 6] = 0u;
    st->whi[(t + 1) % 6] = last;
    st->flo[st->epoch & 1u] = 0u;
    st->fhi[st->epoch & 1u] = last;
    st->wlo[(t + 5) % 6] = 0xFFFFFFFFu;
    st->whi[(t + 5) % 6] = 0u;
  }
  st->dense_bin = 0;
  st->iter = t + 1;
  st->tau = tau;
  st->far_min = rf;
  st->split = split;
  st->stop = stop;
}

__global__ void k_stamp(unsigned long long* p) {
  unsigned long long ns;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ns));
  *p = ns;
}

__global__ void k_sssp_init(uint32_t* __restrict__ dist, const int32_t* __restrict__ slots, int nslots,
                            uint32_t* __restrict__ bm0) {
  // all copies of the source start at 0 (P@28609: copies begin equal)
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  for (int i = 0; i < nslots; i++) {
    const int32_t s = slots[i];
    dist[s] = 0;
    bm0[s >> 5] |= 1u << (s & 31);
  }
}

// static chunk list of heavy rows: chunk count per row, then fill
__global__ void k_heavy_chunks_count(const uint32_t* __restrict__ rp, int64_t n, uint32_t* __restrict__ cnt) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t d = rp[v + 1] - rp[v];
    cnt[v] = d > HEAVY_DEG ? (d + HCHUNK - 1) / HCHUNK : 0u;
  }
}
__global__ void k_heavy_chunks_fill(const uint32_t* __restrict__ rp, int64_t n, const uint32_t* __restrict__ off,
                                    int32_t* __restrict__ hrow, uint32_t* __restrict__ hstart, int64_t row_base = 0) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t d = rp[v + 1] - rp[v];
    if (d <= HEAVY_DEG) continue;
    const uint32_t k = (d + HCHUNK - 1) / HCHUNK, o = off[v];
    for (uint32_t i = 0; i < k; i++) {
      hrow[o + i] = (int32_t)(row_base + v);
      hstart[o + i] = rp[v] + i * HCHUNK;
    }
  }
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
  if (g->default_src >= 0) return g->default_src;   // the canonical input never changes
  Ctx* c = g->ctx;
  DBuf b;
  b.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(b.p, 0, 8, c->stream));
  if (g->n) k_argmax_deg<<<grid_for(c, g->n), 256, 0, c->stream>>>(g->in_rp.as<int64_t>(), g->n,
                                                                   b.as<unsigned long long>());
  unsigned long long h = 0;
  CUDA_OK(cudaMemcpyAsync(&h, b.p, 8, cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  g->default_src = (int64_t)(0xffffffffull - (h & 0xffffffffull));
  return g->default_src;
}

// ---------------------------------------------------------------- driver

void ensure_tpv(gx_graph* g);                                                                  // tpv.cu
void ensure_vns(gx_graph* g);                                                                  // tpv.cu

// Near-far bucket width: a multiple of the mean edge weight scaled down by the
// mean degree (delta-stepping's Delta ~ w / d heuristic), at least 1.
// (the input graph's maximum weight: added 2-hop edges must not change Delta)
static unsigned sssp_delta(const gx_graph* g) {
  const DevGraph& d = g->dg;
  if (d.n_slots == 0 || d.m_slots == 0) return 0u;
  const double avg_deg = (double)g->m / (double)std::max<int64_t>(1, g->n);
  const double avg_w = 0.5 * (1.0 + (double)g->max_w);
  double delta = 8.0 * avg_w / std::max(1.0, avg_deg);
  // sparse, high-diameter graphs (road grids, ~2.5 arcs/vertex) need ~10^4
  // iterations at any bucket width, and each costs ~15 us of barriers and
  // frontier scans: there wide buckets win (road 4900^2, persistent loop:
  // Delta 160 -> 334 ms, 1000 -> 198, 3000 -> 171, 10^4 -> 161, profiles/r1b)
  if (avg_deg < 4.0) delta *= 64.0;
  return (unsigned)std::max(1.0, delta);
}

__global__ void k_adj_wmax(const uint2* __restrict__ adj, int64_t m, unsigned int* __restrict__ out) {
  unsigned int mx = 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
    mx = max(mx, adj[e].y);
  mx = warp_max_u32(mx);
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(out, mx);
}
__global__ void k_adj_pack(const uint2* __restrict__ adj, int64_t m, uint32_t wb, uint32_t* __restrict__ out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
    const uint2 v = adj[e];
    out[e] = (v.x << wb) | v.y;
  }
}

// {dst, w} packed into one u32 when the slot ids and the largest weight fit
// (RMAT-24: 24 + 7 bits): the relaxation stream halves (8 -> 4 B per edge)
static void ensure_packed_adj(gx_graph* g) {
  DevGraph& d = g->dg;
  if (d.adjp_tried) return;
  d.adjp_tried = true;
  if (getenv("GX_SSSP_NO_PACK") || d.m_slots == 0) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  unsigned int wmax = 0;
  if (d.identity) {
    wmax = d.max_w;   // measured at upload
  } else {
    DBuf mx;
    mx.alloc(c, 4);
    CUDA_OK(cudaMemsetAsync(mx.p, 0, 4, s));
    k_adj_wmax<<<grid_for(c, d.m_slots), 256, 0, s>>>(d.adj.as<uint2>(), d.m_slots, mx.as<unsigned int>());
    CUDA_OK(cudaMemcpyAsync(&wmax, mx.p, 4, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
  }
  uint32_t wb = 1;
  while (wb < 32 && (wmax >> wb)) wb++;
  if (wb >= 16 || d.n_slots > (int64_t(1) << (32 - wb))) return;
  d.adjp.alloc(c, sizeof(uint32_t) * d.m_slots);
  k_adj_pack<<<grid_for(c, d.m_slots), 256, 0, s>>>(d.adj.as<uint2>(), d.m_slots, wb, d.adjp.as<uint32_t>());
  CUDA_OK(cudaGetLastError());
  d.adjp_wbits = wb;
}

// light / heavy split of the packed rows at bucket width delta: each row is
// stably partitioned into its light edges (w < delta) then its heavy ones
// (warp per row, ballot ranks), lend[u] = end of the light part.  The order
// of a row's edges does not change the SSSP fixed point.
__global__ void k_adj_lh(const uint32_t* __restrict__ rp, const uint32_t* __restrict__ in, uint32_t* __restrict__ out,
                         uint32_t* __restrict__ lend, int64_t n, uint32_t delta, uint32_t wb) {
  const unsigned lane = lane_id(), lt = (1u << lane) - 1u;
  const uint32_t wm = (1u << wb) - 1u;
  for (int64_t u = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; u < n;
       u += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t a = rp[u], b = rp[u + 1];
    uint32_t nl = 0;
    for (uint32_t e = a + lane; e - lane < b; e += 32)
      nl += __popc(__ballot_sync(FULL, e < b && (in[e] & wm) < delta));
    uint32_t li = a, hi = a + nl;
    for (uint32_t e = a + lane; e - lane < b; e += 32) {
      const bool ok = e < b;
      const uint32_t v = ok ? in[e] : 0u;
      const bool light = ok && (v & wm) < delta;
      const unsigned bl = __ballot_sync(FULL, light), bh = __ballot_sync(FULL, ok && !light);
      if (light) out[li + __popc(bl & lt)] = v;
      else if (ok) out[hi + __popc(bh & lt)] = v;
      li += __popc(bl);
      hi += __popc(bh);
    }
    if (lane == 0) lend[u] = a + nl;
  }
}

static void ensure_lh(gx_graph* g, uint32_t delta) {
  DevGraph& d = g->dg;
  if (d.lh_lend.p && d.lh_delta == delta) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DBuf out;
  out.alloc(c, sizeof(uint32_t) * d.m_slots);
  if (!d.lh_lend.p) d.lh_lend.alloc(c, sizeof(uint32_t) * std::max<int64_t>(1, d.n_slots));
  k_adj_lh<<<c->num_sms * 8, 256, 0, s>>>(d.rp.as<uint32_t>(), d.adjp.as<uint32_t>(), out.as<uint32_t>(),
                                          d.lh_lend.as<uint32_t>(), d.n_slots, delta, d.adjp_wbits);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));
  d.adjp = std::move(out);
  d.lh_delta = delta;
}

static void ensure_heavy_chunks(gx_graph* g) {
  DevGraph& d = g->dg;
  if (d.hc_row.p) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  const int64_t ns = d.n_slots;
  DBuf cnt, off, tmp;
  cnt.alloc(c, sizeof(uint32_t) * (ns + 1));
  off.alloc(c, sizeof(uint32_t) * (ns + 1));
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * (ns + 1), s));
  k_heavy_chunks_count<<<grid_for(c, ns), 256, 0, s>>>(d.rp.as<uint32_t>(), ns, cnt.as<uint32_t>());
  size_t tb = 0;
  CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt.as<uint32_t>(), off.as<uint32_t>(), ns + 1, s));
  tmp.alloc(c, tb);
  CUDA_OK(cub::DeviceScan::ExclusiveSum(tmp.p, tb, cnt.as<uint32_t>(), off.as<uint32_t>(), ns + 1, s));
  uint32_t nhc = 0;
  CUDA_OK(cudaMemcpyAsync(&nhc, off.as<uint32_t>() + ns, 4, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  d.nhc = nhc;
  d.hc_row.alloc(c, sizeof(int32_t) * std::max<uint32_t>(nhc, 1));
  d.hc_start.alloc(c, sizeof(uint32_t) * std::max<uint32_t>(nhc, 1));
  k_heavy_chunks_fill<<<grid_for(c, ns), 256, 0, s>>>(d.rp.as<uint32_t>(), ns, off.as<uint32_t>(), d.hc_row.as<int32_t>(),
                                                      d.hc_start.as<uint32_t>());
  d.heavy_bm.alloc(c, sizeof(uint32_t) * ((ns + 31) / 32));
  k_heavy_bitmap<<<grid_for(c, ns), 256, 0, s>>>(d.rp.as<uint32_t>(), ns, d.heavy_bm.as<uint32_t>());
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));
}

// ---------------------------------------------------------------- partitioned path (dist.h)
// pointer to element -base of a (device) array, so that a rank-local array of
// rows [lo, hi) is indexed with global row ids u in [lo, hi)
template <class T>
static T* shifted(T* p, int64_t base) {
  return reinterpret_cast<T*>(reinterpret_cast<uintptr_t>(p) - (uintptr_t)(base * (int64_t)sizeof(T)));
}

__global__ void k_rebase_rows(const uint32_t* __restrict__ rp, int64_t lo, int64_t n1, uint32_t* __restrict__ out) {
  const uint32_t b = rp[lo];
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n1; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = rp[lo + i] - b;
}

// Rank-local out-CSR of rows [lo, hi) per rank (all P when `all`, else this
// rank), balanced by out-edges: rebased row offsets, the edge slice packed to
// 4 bytes when ids and weights fit, the heavy-chunk list and heavy bitmap.
static RankLayouts& ensure_sssp_ranks(gx_graph* g, int P, bool all) {
  DevGraph& d = g->dg;
  RankLayouts& L = d.rk_sssp;
  Ctx* c = g->ctx;
  const int want_rank = all ? -1 : c->rank;
  if (L.P == P && L.rank == want_rank) return L;
  L = RankLayouts();
  cudaStream_t s = c->stream;
  const int64_t n = d.n_slots;
  std::vector<uint32_t> hrp(n + 1);
  CUDA_OK(cudaMemcpyAsync(hrp.data(), d.rp.p, sizeof(uint32_t) * (n + 1), cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  L.bounds = partition_rows(std::vector<int64_t>(hrp.begin(), hrp.end()), n, P, PRW_ALIGN);
  L.P = P;
  L.rank = want_rank;
  // packing width: the slot graph's largest weight
  unsigned int wmax = d.max_w;
  if (!d.identity) {
    DBuf mx;
    mx.alloc(c, 4);
    CUDA_OK(cudaMemsetAsync(mx.p, 0, 4, s));
    if (d.m_slots) k_adj_wmax<<<grid_for(c, d.m_slots), 256, 0, s>>>(d.adj.as<uint2>(), d.m_slots, mx.as<unsigned int>());
    CUDA_OK(cudaMemcpyAsync(&wmax, mx.p, 4, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
  }
  uint32_t wb = 1;
  while (wb < 32 && (wmax >> wb)) wb++;
  const bool pack = !getenv("GX_SSSP_NO_PACK") && wb < 16 && n <= (int64_t(1) << (32 - wb));
  for (int p = 0; p < P; p++) {
    if (!all && p != c->rank) continue;
    RankSlice sl;
    sl.lo = L.bounds[p];
    sl.hi = L.bounds[p + 1];
    const int64_t nl = sl.hi - sl.lo;
    const int64_t e0 = hrp[sl.lo];
    sl.m = (int64_t)hrp[sl.hi] - e0;
    sl.rp.alloc(c, sizeof(uint32_t) * (nl + 1));
    k_rebase_rows<<<grid_for(c, nl + 1), 256, 0, s>>>(d.rp.as<uint32_t>(), sl.lo, nl + 1, sl.rp.as<uint32_t>());
    if (pack) {
      sl.adjp.alloc(c, sizeof(uint32_t) * std::max<int64_t>(sl.m, 1));
      if (sl.m) k_adj_pack<<<grid_for(c, sl.m), 256, 0, s>>>(d.adj.as<uint2>() + e0, sl.m, wb, sl.adjp.as<uint32_t>());
      sl.wbits = wb;
    } else {
      sl.adj.alloc(c, sizeof(uint2) * std::max<int64_t>(sl.m, 1));
      if (sl.m)
        CUDA_OK(cudaMemcpyAsync(sl.adj.p, d.adj.as<uint2>() + e0, sizeof(uint2) * sl.m, cudaMemcpyDeviceToDevice, s));
    }
    // heavy chunks of the local rows (hc_row global, hc_start local edge index)
    DBuf cnt, off, tmp;
    cnt.alloc(c, sizeof(uint32_t) * (nl + 1));
    off.alloc(c, sizeof(uint32_t) * (nl + 1));
    CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * (nl + 1), s));
    if (nl) k_heavy_chunks_count<<<grid_for(c, nl), 256, 0, s>>>(sl.rp.as<uint32_t>(), nl, cnt.as<uint32_t>());
    size_t tb = 0;
    CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt.as<uint32_t>(), off.as<uint32_t>(), nl + 1, s));
    tmp.alloc(c, tb);
    CUDA_OK(cub::DeviceScan::ExclusiveSum(tmp.p, tb, cnt.as<uint32_t>(), off.as<uint32_t>(), nl + 1, s));
    uint32_t nhc = 0;
    CUDA_OK(cudaMemcpyAsync(&nhc, off.as<uint32_t>() + nl, 4, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    sl.nhc = nhc;
    sl.hc_row.alloc(c, sizeof(int32_t) * std::max<uint32_t>(nhc, 1));
    sl.hc_start.alloc(c, sizeof(uint32_t) * std::max<uint32_t>(nhc, 1));
    if (nl)
      k_heavy_chunks_fill<<<grid_for(c, nl), 256, 0, s>>>(sl.rp.as<uint32_t>(), nl, off.as<uint32_t>(),
                                                         sl.hc_row.as<int32_t>(), sl.hc_start.as<uint32_t>(), sl.lo);
    sl.heavy.alloc(c, sizeof(uint32_t) * std::max<int64_t>((nl + 31) / 32, 1));
    if (nl) k_heavy_bitmap<<<grid_for(c, nl), 256, 0, s>>>(sl.rp.as<uint32_t>(), nl, sl.heavy.as<uint32_t>());
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaStreamSynchronize(s));
    L.r.push_back(std::move(sl));
  }
  return L;
}

// after the exchange the owner holds the reduced distances of its rows; a
// row below its last authoritative value joins the next frontier (or the far
// pile when at or above tau) and becomes the new authoritative value
__global__ void k_frontier_apply(const uint32_t* __restrict__ dist, uint32_t* __restrict__ dauth, SsspAux ax,
                                 SsspState* __restrict__ st, int64_t lo, int64_t hi) {
  if (st->stop) return;
  uint32_t* bm_next = ax.bm[(st->iter + 1) % 3];
  const uint32_t tau = st->tau;
  uint32_t my_min = INF, my_push = 0;
  const int64_t w_lo = lo >> 5, w_hi = (hi + 31) >> 5;   // lo is 32-aligned
  for (int64_t w = w_lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < w_hi; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t near = 0, far = 0;
    for (int b = 0; b < 32; b++) {
      const int64_t v = w * 32 + b;
      if (v >= hi) break;
      const uint32_t nd = dist[v];
      if (nd >= dauth[v - lo]) continue;
      dauth[v - lo] = nd;
      if (nd < tau) {
        near |= 1u << b;
      } else {
        far |= 1u << b;
        my_min = min(my_min, nd);
      }
    }
    if (near) bm_next[w] |= near;
    if (far) ax.far[w] |= far;
    my_push += __popc(near);
  }
  flush_counters(st, st->iter, 0, 0, my_push, my_min);
}

// the merge changed group slots on every rank identically: their new values
// become the owners' authoritative values
__global__ void k_auth_groups(const uint32_t* __restrict__ dist, uint32_t* __restrict__ dauth,
                              const int32_t* __restrict__ gslots, int64_t nslots, int64_t lo, int64_t hi,
                              const SsspState* __restrict__ st) {
  if (st->stop) return;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nslots; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = gslots[i];
    if (v >= lo && v < hi) dauth[v - lo] = dist[v];
  }
}

__global__ void k_init_auth(const uint32_t* __restrict__ dist, uint32_t* __restrict__ dauth, int64_t lo, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dauth[i] = dist[lo + i];
}

// the frontier counters of iteration t (active, pushed) and the far-pile
// minimum to / from the exchange buffers; a stopped loop leaves both alone
__global__ void k_sssp_xch(SsspState* st, uint32_t* xs, int unpack) {
  if (st->stop) return;
  const unsigned k = st->iter % 3;
  if (!unpack) {
    xs[0] = st->active[k];
    xs[1] = st->pushed[k];
    xs[2] = st->far_min;
  } else {
    st->active[k] = xs[0];
    st->pushed[k] = xs[1];
    st->far_min = xs[2];
  }
}

struct SsspRank {
  DBuf dist, mark, st, dauth, xs;
  SsspAux ax{};
  const uint32_t* rp = nullptr;   // rank-local row offsets, indexed by global row
  const uint2* adj = nullptr;
  int64_t lo = 0, hi = 0;
};

// 1-D partitioned SSSP (dist.h): rank p owns slot rows
// [lo_p, hi_p) (edge-balanced over out-edges) and stores only their out-CSR
// (ensure_sssp_ranks).  Per iteration:
//   sweep   k_sssp_lb over the rank's frontier rows, relaxing into its
//           full-length copy of dist (fire-and-forget red.min)
//   reduce  reduce-scatter(min) of dist onto the owners' ranges -- a rank only
//           ever reads authoritative values of its own rows (the heads of the
//           edges it relaxes); stale copies of other rows are upper bounds,
//           so they can only cost extra pushes.  With replica groups the
//           reduction is an allreduce(min): the §2.4 merge needs every copy
//   apply   the owners turn rows that dropped below their last authoritative
//           value into the next frontier / far pile (no full-vector copy:
//           the authoritative values are rank-local, n/P)
//   counters one sum of (active, pushed) and one min of the far minimum, so
//           every rank takes the same near-far decision; advance / refill
// No host synchronisation inside a batch of check_every iterations.
static void run_sssp_dist(gx_graph* g, const gx_run_opts& o, gx_run_info& info, int P, bool sim, int64_t src,
                          unsigned delta) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  const int64_t ns = d.n_slots, nwords = (ns + 31) / 32;
  RankLayouts& RL = ensure_sssp_ranks(g, P, sim);
  const std::vector<int64_t>& bounds = RL.bounds;
  const int nloc = sim ? P : 1;
  std::vector<SsspRank> R(nloc);
  std::vector<int32_t> srcs{d.identity ? (int32_t)src : g->sg.owner_slot[src]};
  if (!d.identity)
    for (int64_t sl = 0; sl < g->sg.n_slots; sl++)
      if (g->sg.kind[sl] == REPLICA && g->sg.slot_to_orig[sl] == src) srcs.push_back((int32_t)sl);
  DBuf dsrc;
  dsrc.alloc(c, sizeof(int32_t) * srcs.size());
  CUDA_OK(cudaMemcpyAsync(dsrc.p, srcs.data(), sizeof(int32_t) * srcs.size(), cudaMemcpyHostToDevice, s));
  SsspState init;
  std::memset(&init, 0, sizeof(init));
  init.delta = delta;
  init.tau = delta ? delta : INF;
  init.far_min = INF;
  init.far3[0] = init.far3[1] = init.far3[2] = INF;
  init.merge_every = 1;
  init.do_merge = 1;
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  for (int p = 0; p < nloc; p++) {
    SsspRank& K = R[p];
    const RankSlice& sl = RL.r[p];
    DBuf& dist = p == 0 ? r.dist : K.dist;
    DBuf& mark = p == 0 ? r.mark : K.mark;
    DBuf& st = p == 0 ? r.st : K.st;
    dist.alloc(c, sizeof(uint32_t) * ns);
    mark.alloc(c, sizeof(uint32_t) * 4 * nwords);
    st.alloc(c, sizeof(SsspState));
    K.lo = sl.lo;
    K.hi = sl.hi;
    K.dauth.alloc(c, sizeof(uint32_t) * std::max<int64_t>(K.hi - K.lo, 1));
    K.xs.alloc(c, sizeof(uint32_t) * 4);
    for (int i = 0; i < 3; i++) K.ax.bm[i] = mark.as<uint32_t>() + i * nwords;
    K.ax.far = mark.as<uint32_t>() + 3 * nwords;
    K.ax.heavy = shifted(sl.heavy.as<uint32_t>(), K.lo >> 5);
    K.ax.nwords = nwords;
    K.ax.hc_row = sl.hc_row.as<int32_t>();
    K.ax.hc_start = sl.hc_start.as<uint32_t>();
    K.ax.nhc = sl.nhc;
    K.ax.adjp = sl.adjp.p ? sl.adjp.as<uint32_t>() : nullptr;
    K.ax.wbits = sl.wbits;
    K.rp = shifted(sl.rp.as<uint32_t>(), K.lo);
    K.adj = sl.adj.p ? sl.adj.as<uint2>() : nullptr;
    CUDA_OK(cudaMemsetAsync(dist.p, 0xFF, sizeof(uint32_t) * ns, s));
    CUDA_OK(cudaMemsetAsync(mark.p, 0, sizeof(uint32_t) * 4 * nwords, s));
    CUDA_OK(cudaMemcpyAsync(st.p, &init, sizeof(SsspState), cudaMemcpyHostToDevice, s));
    k_sssp_init<<<1, 32, 0, s>>>(dist.as<uint32_t>(), dsrc.as<int32_t>(), (int)srcs.size(), K.ax.bm[0]);
    if (K.hi > K.lo) k_init_auth<<<grid_for(c, K.hi - K.lo), 256, 0, s>>>(dist.as<uint32_t>(), K.dauth.as<uint32_t>(), K.lo, K.hi - K.lo);
  }
  auto D = [&](int p) { return (p == 0 ? r.dist : R[p].dist).as<uint32_t>(); };
  auto S = [&](int p) { return (p == 0 ? r.st : R[p].st).as<SsspState>(); };
  Exch X;
  X.c = c;
  X.P = P;
  X.sim = sim;
  int occ = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sssp_lb, 256, 0));
  const int grid_lb = std::max(1, occ) * c->num_sms;
  const int grid_local = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_tiles + 7) / 8, (int64_t)c->num_sms * 8));   // a warp per tile
  const int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_groups + 7) / 8, (int64_t)c->num_sms * 8));
  const bool merge_min = g->knobs.merge_op == GX_MERGE_MIN;
  std::vector<void*> dl, xsl, xml;
  for (int p = 0; p < nloc; p++) {
    dl.push_back(D(p));
    xsl.push_back(R[p].xs.p);
    xml.push_back(R[p].xs.as<uint32_t>() + 2);
  }
  const int batch = std::max(1, o.check_every);
  int launches = 0;
  SsspState hst;
  for (;;) {
    for (int it = 0; it < batch; it++) {
      for (int p = 0; p < nloc; p++) {
        k_sssp_lb<<<grid_lb, 256, 0, s>>>(R[p].rp, R[p].adj, D(p), R[p].ax, S(p), R[p].lo, R[p].hi);
        launches++;
        if (d.n_tiles && g->knobs.smem) {
          k_sssp_local<<<grid_local, 256, 0, s>>>(d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(), d.t_eptr.as<int32_t>(),
                                                  d.t_edges.as<uint2>(), d.t_iters.as<int32_t>(), d.n_tiles, D(p), R[p].ax,
                                                  S(p), nullptr, nullptr);
          launches++;
        }
      }
      if (d.n_groups) X.allreduce(dl, ns, Dt::U32, Op::MIN);     // the merge reads every copy
      else X.reduce_scatterv(dl, bounds, Dt::U32, Op::MIN);      // owners' ranges only
      for (int p = 0; p < nloc; p++) {
        k_frontier_apply<<<grid_for(c, (R[p].hi - R[p].lo + 31) / 32 + 1), 256, 0, s>>>(D(p), R[p].dauth.as<uint32_t>(),
                                                                                         R[p].ax, S(p), R[p].lo, R[p].hi);
        launches++;
        if (d.n_groups) {
          k_sssp_merge<<<grid_merge, 256, 0, s>>>(d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), d.g_in_ptr.as<int32_t>(),
                                                  d.g_in.as<uint2>(), d.n_groups, merge_min ? 1 : 0, D(p), R[p].ax, S(p));
          k_auth_groups<<<grid_for(c, d.n_gslots), 256, 0, s>>>(D(p), R[p].dauth.as<uint32_t>(), d.gslots.as<int32_t>(),
                                                                d.n_gslots, R[p].lo, R[p].hi, S(p));
          launches += 2;
        }
        k_sssp_xch<<<1, 1, 0, s>>>(S(p), R[p].xs.as<uint32_t>(), 0);
        launches++;
      }
      X.allreduce(xsl, 2, Dt::U32, Op::SUM);   // active, pushed of iteration t
      X.allreduce(xml, 1, Dt::U32, Op::MIN);   // far-pile minimum: the same bucket decision everywhere
      for (int p = 0; p < nloc; p++) {
        k_sssp_xch<<<1, 1, 0, s>>>(S(p), R[p].xs.as<uint32_t>(), 1);
        k_sssp_advance<<<1, 1, 0, s>>>(S(p), o.max_iters);
        k_sssp_split<<<grid_for(c, nwords), 256, 0, s>>>(D(p), R[p].ax, S(p), R[p].lo, R[p].hi);
        launches += 3;
      }
    }
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaMemcpyAsync(&hst, S(0), sizeof(SsspState), cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (hst.stop) break;
  }
  // result: each rank's authoritative rows -> every rank
  for (int p = 0; p < nloc; p++)
    if (R[p].hi > R[p].lo)
      CUDA_OK(cudaMemcpyAsync(D(p) + R[p].lo, R[p].dauth.p, sizeof(uint32_t) * (R[p].hi - R[p].lo),
                              cudaMemcpyDeviceToDevice, s));
  X.allgatherv(dl, bounds, Dt::U32);
  unsigned long long edges = 0;
  for (int p = 0; p < nloc; p++) {
    SsspState h;
    CUDA_OK(cudaMemcpyAsync(&h, S(p), sizeof(SsspState), cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    edges += h.edges;
  }
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = (int32_t)hst.iter;
  info.converged = hst.stop == 1;
  info.loop_ms = ms;
  info.edges_scanned = (int64_t)edges;                 // this rank's relaxations (all simulated ranks when sim)
  info.vertices_active = (int64_t)hst.act_total;       // global (the counters are reduced)
  info.bytes_model = 12 * (int64_t)edges + 14 * (int64_t)hst.act_total / (sim ? 1 : P);
  info.kernel_launches = launches;
  info.mapping_used = GX_MAP_LB;
  r.have[GX_SSSP] = true;
}

// GX_SSSP_WINCHECK=1: bits left in the far pile / the three frontier bitmaps
// after the loop (the far pile must be empty at convergence)
__global__ void k_popc_words(const uint32_t* __restrict__ w, int64_t nwords, unsigned long long* __restrict__ out) {
  unsigned long long c = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nwords; i += (int64_t)gridDim.x * blockDim.x)
    c += __popc(w[i]);
  c = warp_sum_u64(c);
  if (lane_id() == 0 && c) atomicAdd(out, c);
}

static void run_sssp_impl(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  const int64_t src = o.source < 0 ? default_source(g) : o.source;
  GX_CHECK_ARG(g->n > 0, "empty graph");
  GX_CHECK_ARG(src >= 0 && src < g->n, "source out of range");
  // the bound uses the INPUT graph's weights: an added edge stands for a path
  // at least as long (sum rule) or is lighter than both hops (max / mean
  // rules), so no distance exceeds (n-1) * max w of the input
  // R51: every du + w saturates at 2^32-2, which is never a shortest distance
  // when all true distances are below it; run_sssp checks the result for it
  // afterwards instead of refusing graphs whose static bound (n-1)*max(w)
  // exceeds 32 bits (RMAT-26: 6.7e9, true distances < 1000)
  const bool sim = c->world == 1 && o.sim_ranks > 1;
  const int P = sim ? o.sim_ranks : c->world;
  if (P > 1) {
    GX_CHECK_ARG(P <= 8, "at most 8 ranks");
    GX_CHECK_ARG(o.mapping != GX_MAP_TPV && o.mapping != GX_MAP_VNS, "the partitioned path uses the LB mapping");
    GX_CHECK_ARG(o.merge_every == 1 || !d.n_groups, "the partitioned path merges after every iteration");
    unsigned delta = sssp_delta(g);
    if (const char* e = getenv("GX_SSSP_DELTA")) delta = (unsigned)std::max(0, atoi(e));
    run_sssp_dist(g, o, info, P, sim, src, delta);
    return;
  }
  int mapping = o.mapping == GX_MAP_PB ? GX_MAP_LB : o.mapping;   // PB is a PageRank mapping
  // AUTO = LB, measured fastest on every configuration incl. the §2 / §4
  // graphs (RMAT-22 §2: LB 2.8 vs TPV 8.9 ms; road §2: 116 vs 1246; uniform
  // §4: 4.2 vs 14.4; profiles/r2/knobs); TPV = the paper's mapping, on request
  if (mapping == GX_MAP_AUTO) mapping = GX_MAP_LB;
  if (mapping == GX_MAP_TPV) ensure_tpv(g);
  if (mapping == GX_MAP_VNS) ensure_vns(g);
  ensure_heavy_chunks(g);
  const int64_t ns = d.n_slots;
  const int64_t nwords = (ns + 31) / 32;
  r.dist.alloc(c, sizeof(uint32_t) * ns);
  r.mark.alloc(c, sizeof(uint32_t) * 6 * nwords);   // frontier bitmaps bm[0..2] + far pile + pend[0..1]
  r.st.alloc(c, sizeof(SsspState));
  SsspState* st = r.st.as<SsspState>();
  SsspAux ax{};
  for (int i = 0; i < 3; i++) ax.bm[i] = r.mark.as<uint32_t>() + i * nwords;
  ax.far = r.mark.as<uint32_t>() + 3 * nwords;
  ax.heavy = d.heavy_bm.as<uint32_t>();
  ax.nwords = nwords;
  ax.hc_row = d.hc_row.as<int32_t>();
  ax.hc_start = d.hc_start.as<uint32_t>();
  ax.nhc = d.nhc;
  if (mapping == GX_MAP_LB) {
    ensure_packed_adj(g);
    ax.adjp = d.adjp.as<uint32_t>();
    ax.wbits = d.adjp_wbits;
  }
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

  // light / heavy split (persistent LB loop, exact mode on packed rows: no §3
  // tiles or §2 merges, which move distances outside the sweeps); the layout
  // is built once per bucket width, outside the timed region.  Off unless
  // GX_SSSP_LH=1: measured on RMAT-24 it relaxes 374M edges instead of 451M but
  // takes 72 iterations instead of 57 and 5.33 ms instead of 5.10 (Delta 12-100
  // all slower than the default without it; profiles/r1e/lh_sweep.txt)
  unsigned hst_delta = mapping == GX_MAP_LB ? sssp_delta(g) : 0u;
  if (const char* e = getenv("GX_SSSP_DELTA")) hst_delta = (unsigned)std::max(0, atoi(e));
  bool want_lh = false;
  {
    const char* lhe = getenv("GX_SSSP_LH");
    const char* pe0 = getenv("GX_SSSP_PERSIST");
    const char* be0 = getenv("GX_SSSP_BLOCK");
    want_lh = mapping == GX_MAP_LB && ax.adjp && hst_delta > 0 && !(d.n_tiles && g->knobs.smem) && !d.n_groups &&
              (lhe && atoi(lhe) != 0) && !(pe0 && atoi(pe0) == 0) && !(be0 && atoi(be0) != 0) &&
              !(o.profile && getenv("GX_SSSP_TRACE"));
    if (want_lh) {
      ensure_lh(g, hst_delta);
      ax.adjp = d.adjp.as<uint32_t>();   // the partitioned copy replaced the buffer
    }
  }
  // blocked dense relaxation for refills that carry most of the edges
  // (persistent LB loop on a graph without merges, tiles or the light/heavy
  // split; weights must fit the layout's 8-bit array).  GX_SSSP_DENSE = the
  // fraction of the slots a refill must move (default 0.45; 0 = off).  The
  // dense pass costs one streaming pass over all edges (RMAT-24: scatter 0.49
  // + gather 0.43 ms) against ~140 G relaxations/s for the LB sweep, so it
  // pays once a refill carries about half of the edges: RMAT-24's first
  // refill moves 51 % of the slots with 76 % of the edges (4.85 -> 4.49 ms);
  // uniform and RMAT-22 refills at 40 % lost 0.4 / 0.13 ms
  // (profiles/r2/sssp_dense_sweep.txt)
  // When dist no longer fits the L2 (RMAT-26: 256 MB), the LB sweep's gathers
  // go to DRAM and the streamed pass pays from smaller refills: RMAT-26 at
  // 0.25-0.3: 30.1 -> 26.3 ms (profiles/r2/sssp_dense_rmat26_farscan.txt)
  double dense_frac = (double)d.n_slots * 4.0 > 96.0 * (1 << 20) ? 0.25 : 0.45;
  if (const char* e = getenv("GX_SSSP_DENSE")) dense_frac = atof(e);
  // (with §3 tiles the dense iteration skips the local pass, schedule-only by
  // E1; with replica groups it merges after the gather, every iteration only)
  const bool dense_ok = mapping == GX_MAP_LB && dense_frac > 0.0 && (!d.n_groups || o.merge_every == 1) &&
                        !want_lh && d.max_w <= 0xffffu && d.m_slots > 0 && !getenv("GX_SSSP_BLOCK") &&
                        !(o.profile && getenv("GX_SSSP_TRACE"));
  SsspPb spb{};
  bool dense_on = dense_ok;
  if (dense_on) dense_on = ensure_pb_w(g);   // false after an asynchronous upload's structure-only layout
  if (dense_on) {
    spb.q = d.pr_pb.q.as<uint32_t>();
    spb.src_loc = d.pr_pb.src_loc.as<uint16_t>();
    spb.dst_loc = d.pr_pb.dst_loc.as<uint16_t>();
    spb.w16 = d.pb_w16.as<uint16_t>();
    spb.val = d.pr_pb.val.as<uint32_t>();
    spb.nb = d.pr_pb.nb;
    CUDA_OK(cudaFuncSetAttribute(k_sssp_pb_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (PB_R + 8) * 4));
    CUDA_OK(cudaFuncSetAttribute(k_sssp_pb_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, PB_R * 4));
  }
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  CUDA_OK(cudaMemsetAsync(r.dist.p, 0xFF, sizeof(uint32_t) * ns, s));
  CUDA_OK(cudaMemsetAsync(r.mark.p, 0, sizeof(uint32_t) * 6 * nwords, s));
  bool win_h = false;
  {
    // near-far bucket width (LB mapping only; 0 = plain frontier Bellman-Ford)
    static SsspState init;
    std::memset(&init, 0, sizeof(init));
    unsigned delta = mapping == GX_MAP_LB ? sssp_delta(g) : 0u;
    if (const char* e = getenv("GX_SSSP_DELTA")) delta = (unsigned)std::max(0, atoi(e));
    init.delta = delta;
    init.tau = delta ? delta : INF;
    init.far_min = INF;
  init.far3[0] = init.far3[1] = init.far3[2] = INF;
    init.merge_every = d.n_groups ? (unsigned)o.merge_every : 1u;
    init.do_merge = init.merge_every == 1 ? 1u : 0u;
    // frontier windows (honoured by the persistent LB loop only): off when
    // merges, §3 tiles, the light/heavy split or the block mode set bits
    // outside the sweep's bookkeeping.  On by default for high-diameter graphs
    // (avg_deg < 4) of >= 4M slots, where a bucket's frontier covers a thin
    // band of the id space (road 4900^2: 157 -> 143 ms; RMAT-24 / uniform
    // +1.5 %, road 1024^2 +9 %: profiles/r2/sssp_window_sweep.txt);
    // GX_SSSP_WINDOW=0 / 1 forces them off / on
    const char* we = getenv("GX_SSSP_WINDOW");
    const bool win_ok = mapping == GX_MAP_LB && !d.n_groups && !(d.n_tiles && g->knobs.smem) && !want_lh &&
                        !getenv("GX_SSSP_BLOCK");
    const bool win_auto = (double)g->m < 4.0 * (double)std::max<int64_t>(1, g->n) && d.n_slots >= (int64_t(1) << 22);
    init.win_on = win_ok && (we ? atoi(we) != 0 : win_auto) ? 1u : 0u;
    win_h = init.win_on != 0;
    init.wlo[0] = 0xFFFFFFFFu;
    for (int32_t sv : srcs) {
      init.wlo[0] = std::min(init.wlo[0], (unsigned)(sv >> 5));
      init.whi[0] = std::max(init.whi[0], (unsigned)(sv >> 5));
    }
    for (int i = 1; i < 6; i++) init.wlo[i] = 0xFFFFFFFFu;
    init.flo[0] = init.flo[1] = 0xFFFFFFFFu;
    CUDA_OK(cudaMemcpyAsync(r.st.p, &init, sizeof(SsspState), cudaMemcpyHostToDevice, s));
  }
  k_sssp_init<<<1, 32, 0, s>>>(r.dist.as<uint32_t>(), dsrc.as<int32_t>(), (int)srcs.size(), ax.bm[0]);
  CUDA_OK(cudaGetLastError());
  int launches = 4;

  int occ = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sssp_lb, 256, 0));
  const int grid_lb = std::max(1, occ) * c->num_sms;
  int occt = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occt, k_sssp_tpv, 256, 0));
  const int grid_tpv = std::max(1, occt) * c->num_sms;
  const int grid_local = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_tiles + 7) / 8, (int64_t)c->num_sms * 8));   // a warp per tile
  const int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_groups + 7) / 8, (int64_t)c->num_sms * 8));
  const bool merge_min = g->knobs.merge_op == GX_MERGE_MIN;
  const int grid_split = grid_for(c, nwords);

  KTimer kt(o.profile != 0, s);
  auto one_iter = [&](int& nl) {
    kt.begin();
    if (mapping == GX_MAP_TPV) {
      k_sssp_tpv<<<grid_tpv, 256, 0, s>>>(d.tpv_lane_row.as<int32_t>(), d.tpv_out_len.as<uint32_t>(),
                                          d.tpv_out_off.as<uint64_t>(), d.tpv_out_slab.as<uint2>(), d.tpv_nslices,
                                          r.dist.as<uint32_t>(), ax, st);
      nl++;
    } else if (mapping == GX_MAP_VNS) {
      // the TPV sweep over virtual nodes: lane -> its slot (dist, frontier), slab -> its <= K edges
      k_sssp_tpv<<<grid_tpv, 256, 0, s>>>(d.vns_lane_slot.as<int32_t>(), d.vns_len.as<uint32_t>(),
                                          d.vns_off.as<uint64_t>(), d.vns_slab.as<uint2>(), d.vns_nslices,
                                          r.dist.as<uint32_t>(), ax, st);
      nl++;
    } else {
      k_sssp_lb<<<grid_lb, 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), r.dist.as<uint32_t>(), ax, st, 0, ns);
      nl++;
    }
    kt.end();
    if (d.n_tiles && g->knobs.smem) {
      k_sssp_tiles_collect<<<grid_for(c, nwords), 256, 0, s>>>(ax, st, d.slot_tile.as<int32_t>(),
                                                               d.tile_mark.as<uint32_t>(), d.tile_list.as<int32_t>());
      k_sssp_local<<<grid_local, 256, 0, s>>>(d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(), d.t_eptr.as<int32_t>(),
                                              d.t_edges.as<uint2>(), d.t_iters.as<int32_t>(), d.n_tiles,
                                              r.dist.as<uint32_t>(), ax, st, d.tile_list.as<int32_t>(),
                                              d.tile_mark.as<uint32_t>());
      nl += 2;
    }
    if (d.n_groups) {
      if (o.merge_every != 1) {
        k_sssp_merge_decide<<<1, 1, 0, s>>>(st);
        nl++;
      }
      k_sssp_merge<<<grid_merge, 256, 0, s>>>(d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), d.g_in_ptr.as<int32_t>(),
                                              d.g_in.as<uint2>(), d.n_groups, merge_min ? 1 : 0, r.dist.as<uint32_t>(),
                                              ax, st);
      nl++;
    }
    k_sssp_advance<<<1, 1, 0, s>>>(st, o.max_iters);
    nl++;
    if (mapping == GX_MAP_LB) {
      k_sssp_split<<<grid_split, 256, 0, s>>>(r.dist.as<uint32_t>(), ax, st, 0, ns);
      nl++;
    }
  };

  const int batch = std::max(1, o.check_every);
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
  // GX_SSSP_TRACE (profile runs): one stderr line per iteration --
  // iteration, frontier size, cumulative edges, tau, far_min, sweep-kernel ms
  const bool trace = o.profile && getenv("GX_SSSP_TRACE");
  // LB mapping: the whole loop as one cooperative launch (k_sssp_persist);
  // GX_SSSP_PERSIST=0 selects the per-kernel loop below (A/B, tracing)
  int occp = 0, coop = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occp, k_sssp_persist, PERSIST_TPB, 0));
  CUDA_OK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, c->device));
  const char* pe = getenv("GX_SSSP_PERSIST");
  const bool persist = mapping == GX_MAP_LB && coop && occp > 0 && !trace && !(pe && atoi(pe) == 0);
  if (persist) {
    SsspLoop L;
    L.rp = d.rp.as<uint32_t>();
    L.adj = d.adj.as<uint2>();
    L.dist = r.dist.as<uint32_t>();
    L.ax = ax;
    L.st = st;
    L.n_slots = ns;
    const bool tiles = d.n_tiles && g->knobs.smem;
    L.tptr = d.t_ptr.as<int32_t>();
    L.tmem = d.t_members.as<int32_t>();
    L.teptr = d.t_eptr.as<int32_t>();
    L.titers = d.t_iters.as<int32_t>();
    L.tedges = d.t_edges.as<uint2>();
    L.ntiles = tiles ? d.n_tiles : 0;
    L.slot_tile = d.slot_tile.as<int32_t>();
    L.tmark = d.tile_mark.as<uint32_t>();
    L.tlist = d.tile_list.as<int32_t>();
    L.gptr = d.gptr.as<int32_t>();
    L.gslots = d.gslots.as<int32_t>();
    L.ginptr = d.g_in_ptr.as<int32_t>();
    L.gin = d.g_in.as<uint2>();
    L.ngroups = d.n_groups;
    L.merge_min = merge_min ? 1 : 0;
    L.cadence = o.merge_every != 1 ? 1 : 0;
    L.max_iters = o.max_iters;
    // early refill (measured, profiles/r2/sssp_early_sweep.txt): at <= 256
    // pushes RMAT-24 4.73 -> 4.55 ms (57 -> 40 iterations), uniform 16M/256M
    // 4.35 -> 4.18, road 4900^2 147 -> 142; >= 1024 refills RMAT's first
    // bucket before it settles (451M -> 841M relaxations)
    L.early = 256;
    if (const char* e = getenv("GX_SSSP_EARLY")) L.early = (unsigned)std::max(0, atoi(e));
    // adaptive window (GX_SSSP_WMUL_CAP = 1 turns it off).  Measured
    // (profiles/r2/sssp_wmul_sweep.txt): RMAT-24 4.66 -> 4.55 ms, uniform
    // 16M/256M 4.69 -> 4.07 ms (cap 8 = cap 64); off for sparse high-diameter
    // graphs (the avg-degree < 4 rule of sssp_delta), whose buckets are always
    // small wavefronts: road 4900^2 151 -> 175-187 ms with it
    L.small_refill = (unsigned long long)std::max<int64_t>(1, ns / 256);
    const double avg_deg = (double)g->m / (double)std::max<int64_t>(1, g->n);
    L.wmul_cap = avg_deg < 4.0 ? 1u : 8u;
    if (const char* e = getenv("GX_SSSP_WMUL_CAP")) L.wmul_cap = (unsigned)std::max(1, atoi(e));
    // block-local mode when most edges stay inside the CTA id blocks and rows
    // are short (thread-per-slot relaxation); GX_SSSP_BLOCK=0/1 overrides
    const int64_t gridp = (int64_t)occp * c->num_sms;
    const int64_t B = ((ns + gridp - 1) / gridp + 31) / 32 * 32;
    L.block_rows = 0;
    const char* be = getenv("GX_SSSP_BLOCK");
    // (the locality count costs ~2 ms on RMAT-24: only when the mode is asked for)
    if (B <= BLK_MAX && d.m_slots > 0 && be && atoi(be) != 0) {
      if (d.blk_rows != B) {
        DBuf cnt;
        cnt.alloc(c, 16);
        CUDA_OK(cudaMemsetAsync(cnt.p, 0, 16, s));
        k_block_locality<<<grid_for(c, ns), 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), ns, B,
                                                        cnt.as<unsigned long long>());
        unsigned long long h[2];
        CUDA_OK(cudaMemcpyAsync(h, cnt.p, 16, cudaMemcpyDeviceToHost, s));
        CUDA_OK(cudaStreamSynchronize(s));
        d.blk_rows = B;
        d.blk_local = (double)h[0] / (double)d.m_slots;
        d.blk_maxdeg = (int64_t)h[1];
      }
      // experimental: off unless GX_SSSP_BLOCK=1 (road 4900^2: 326 ms at the
      // default Delta vs 331 for the LB sweep, but 270 vs 198 at Delta 1000 --
      // each local round still pays an L2 round trip per hop)
      const bool want = be ? atoi(be) != 0 && d.blk_maxdeg <= 64 : false;
      if (want) L.block_rows = B;
    }
    // far pile by scan (sssp_split_dev): no far bitmap, so a relaxation that
    // lands beyond tau issues one reduction (dist) instead of two; the refill
    // reads dist once, coalesced.  Not with windows (a scan of all of dist per
    // refill, ~10^3 refills on a road grid), the light/heavy split or the
    // block mode (they push far bits of their own).  Merges and §3 local passes
    // keep it: every value they lower is pushed into the next near frontier
    // (processed there, at any value), and a value a mean merge raises is at
    // worst processed once more by a later scan -- any relaxation order
    // reaches the same fixed point (E1).  GX_SSSP_FARSCAN=0 keeps the bitmap
    const char* fse = getenv("GX_SSSP_FARSCAN");
    const bool far_scan = !win_h && !want_lh && L.block_rows == 0 && !(fse && atoi(fse) == 0);
    if (far_scan) {
      L.ax.far = nullptr;
      ax.far = nullptr;   // the dense iteration's gather too
    }
    if (want_lh && L.block_rows == 0) {
      L.ax.lend = d.lh_lend.as<uint32_t>();
      L.ax.pend[0] = r.mark.as<uint32_t>() + 4 * nwords;
      L.ax.pend[1] = r.mark.as<uint32_t>() + 5 * nwords;
    }
    // GX_SSSP_PTRACE=1: per-iteration timestamps of the persistent loop (stderr)
    DBuf trace_buf;
    L.trace = nullptr;
    L.trace_cap = 0;
    if (getenv("GX_SSSP_PTRACE")) {
      L.trace_cap = 1 << 16;
      trace_buf.alloc(c, sizeof(unsigned long long) * 4 * (L.trace_cap + 1));
      L.trace = trace_buf.as<unsigned long long>() + 4;
      unsigned long long t0 = 0;
      CUDA_OK(cudaMemsetAsync(trace_buf.p, 0, 32, s));
      (void)t0;
    }
    void* args[] = {&L};
    kt.begin();
    L.dense_edges = dense_on ? (unsigned long long)std::max(1.0, dense_frac * (double)d.n_slots) : 0ull;
    if (L.trace) k_stamp<<<1, 1, 0, s>>>(trace_buf.as<unsigned long long>());
    for (;;) {
      CUDA_OK(cudaLaunchCooperativeKernel((void*)k_sssp_persist, dim3((unsigned)(occp * c->num_sms)), dim3(PERSIST_TPB),
                                          args, 0, s));
      launches += 1;
      CUDA_OK(cudaMemcpyAsync(&hst, st, sizeof(SsspState), cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (hst.stop != 4) break;
      // the refill carries most of the edges: one blocked dense iteration, then
      // the persistent loop resumes (stop = 4 -> the decision -> 0 / 1 / 2)
      const int gs = (int)std::min<int64_t>(spb.nb, (int64_t)c->num_sms * 2);
      const int gg = (int)std::min<int64_t>(spb.nb, (int64_t)c->num_sms);
      cudaEvent_t d0 = nullptr, d1 = nullptr, d2 = nullptr;
      if (L.trace) {
        CUDA_OK(cudaEventCreate(&d0));
        CUDA_OK(cudaEventCreate(&d1));
        CUDA_OK(cudaEventCreate(&d2));
        CUDA_OK(cudaEventRecord(d0, s));
      }
      k_sssp_pb_scatter<<<gs, SPB_THREADS, (PB_R + 8) * 4, s>>>(spb, r.dist.as<uint32_t>(), ax, st, ns);
      if (L.trace) CUDA_OK(cudaEventRecord(d1, s));
      k_sssp_pb_gather<<<gg, SPB_THREADS, PB_R * 4, s>>>(spb, r.dist.as<uint32_t>(), ax, st, ns);
      if (L.trace) {
        CUDA_OK(cudaEventRecord(d2, s));
        CUDA_OK(cudaEventSynchronize(d2));
        float a1 = 0, a2 = 0;
        cudaEventElapsedTime(&a1, d0, d1);
        cudaEventElapsedTime(&a2, d1, d2);
        fprintf(stderr, "sssp-ptrace dense t=%u scatter_us=%.1f gather_us=%.1f\n", hst.iter, 1e3 * a1, 1e3 * a2);
        cudaEventDestroy(d0);
        cudaEventDestroy(d1);
        cudaEventDestroy(d2);
      }
      if (d.n_groups)   // §2.4 confluence of the dense iteration (stop == 4 is still running)
        k_sssp_merge<<<grid_merge, 256, 0, s>>>(d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), d.g_in_ptr.as<int32_t>(),
                                                d.g_in.as<uint2>(), d.n_groups, merge_min ? 1 : 0,
                                                r.dist.as<uint32_t>(), ax, st);
      k_sssp_dense_decide<<<1, 1, 0, s>>>(st, d.m_slots, L.early, o.max_iters, nwords);
      CUDA_OK(cudaGetLastError());
      launches += 3;
      info.dense_iterations++;
      CUDA_OK(cudaMemcpyAsync(&hst, st, sizeof(SsspState), cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      if (hst.stop) break;
    }
    kt.end();
    if (L.trace) {
      const int nt = std::min<int>((int)hst.iter, L.trace_cap);
      std::vector<unsigned long long> h(4 * (nt + 1));
      CUDA_OK(cudaMemcpy(h.data(), trace_buf.p, sizeof(unsigned long long) * h.size(), cudaMemcpyDeviceToHost));
      unsigned long long prev_e = 0;
      for (int t = 0; t < nt; t++) {
        const unsigned long long* r = &h[4 * (t + 1)];
        fprintf(stderr, "sssp-ptrace t=%d us=%.2f act=%llu edges=%llu tau=%llu\n", t, (r[0] - h[4 * t]) * 1e-3, r[2],
                r[1] - prev_e, r[3]);
        prev_e = r[1];
      }
    }
  }
  while (!persist) {
    if (gexec) {
      CUDA_OK(cudaGraphLaunch(gexec, s));
      launches += per_batch_launches;
    } else if (trace) {
      one_iter(launches);
      CUDA_OK(cudaMemcpyAsync(&hst, st, sizeof(SsspState), cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
      float kms = 0;
      cudaEventElapsedTime(&kms, kt.ev[kt.ev.size() - 2], kt.ev.back());
      fprintf(stderr, "sssp-trace t=%u act=%u edges=%llu tau=%u far_min=%u split=%u sweep_ms=%.4f\n", hst.iter - 1,
              hst.active[(hst.iter - 1) % 3], hst.edges, hst.tau, hst.far_min, hst.split, kms);
    } else {
      for (int i = 0; i < batch; i++) one_iter(launches);
    }
    CUDA_OK(cudaGetLastError());
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
  if (getenv("GX_SSSP_WINCHECK")) {
    DBuf cnt;
    cnt.alloc(c, 8 * 4);
    CUDA_OK(cudaMemsetAsync(cnt.p, 0, 32, s));
    for (int i = 0; i < 4; i++)
      k_popc_words<<<grid_for(c, nwords), 256, 0, s>>>(r.mark.as<uint32_t>() + i * nwords, nwords,
                                                       cnt.as<unsigned long long>() + i);
    unsigned long long hc[4];
    CUDA_OK(cudaMemcpyAsync(hc, cnt.p, 32, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    fprintf(stderr, "sssp-wincheck iter=%u bm0=%llu bm1=%llu bm2=%llu far=%llu\n", hst.iter, hc[0], hc[1], hc[2],
            hc[3]);
  }
  // iterations that processed a non-empty frontier
  info.iterations = (int32_t)(hst.stop == 1 ? hst.iter : hst.iter);
  info.converged = hst.stop == 1;
  info.loop_ms = ms;
  info.edges_scanned = (int64_t)hst.edges;
  info.vertices_active = (int64_t)hst.act_total;
  // bytes model: 12 B per relaxed edge ({col,w} 8 + dist gather 4)
  // + 12 B per frontier slot (row_ptr 8 + dist 4)
  info.bytes_model = 12 * (int64_t)hst.edges + 12 * (int64_t)hst.act_total;
  info.kernel_launches = launches;
  info.sweep_launches = kt.launches();
  info.sweep_ms = kt.total_ms();
  // packed edges: {dst, w} in 4 bytes instead of 8
  info.sweep_bytes = ax.adjp ? 8 * (int64_t)hst.edges + 12 * (int64_t)hst.act_total : info.bytes_model;
  info.mapping_used = mapping;
  r.have[GX_SSSP] = true;
}

__global__ void k_sat_check(const uint32_t* __restrict__ dist, int64_t n, unsigned int* __restrict__ flag) {
  bool hit = false;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    hit |= dist[v] == INF - 1;
  if (__syncthreads_or(hit) && threadIdx.x == 0) *flag = 1u;
}

void run_sssp(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  run_sssp_impl(g, o, info);
  // a distance at the saturation value means a path length reached 2^32-2:
  // the uint32 result may be wrong, report it (R51)
  Ctx* c = g->ctx;
  DBuf f;
  f.alloc(c, 4);
  CUDA_OK(cudaMemsetAsync(f.p, 0, 4, c->stream));
  k_sat_check<<<grid_for(c, g->dg.n_slots), 256, 0, c->stream>>>(g->rs.dist.as<uint32_t>(), g->dg.n_slots,
                                                                   f.as<unsigned int>());
  unsigned int h = 0;
  CUDA_OK(cudaMemcpyAsync(&h, f.p, 4, cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  if (h) {
    g->rs.have[GX_SSSP] = false;
    GX_THROW(GX_E_UNSUPPORTED, "a shortest-path length reached 2^32-2: uint32 distances overflow");
  }
}

}  // namespace gx
