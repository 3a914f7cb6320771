// pagerank.cu -- PageRank pull sweeps.
//
// x'_v = (1-d)/N + d * ( sum_{u->v} x_u / D_u  +  dangling / N )
// (reading R35; D = total logical out-degree, so replica copies each divide by
// the vertex's full out-degree and mass is not double counted, Theorem E3).
//
// LB pull = windowed SELL-32 (sell.cu): one CTA per window of PRW rows.  The
// window's light rows were sorted by in-degree into 32-lane slices, so a warp
// reads the j-th in-edge of 32 rows with one coalesced 128-byte load (L2
// evict_first) and every lane accumulates its own row in fp64 from fp32
// contrib gathers (L2 evict_last) with 8 gathers in flight; rows with more
// than PR_HEAVY in-edges are reduced warp-per-row.  Row sums stay in shared
// memory and the PR update of the window (x, delta, next contrib, dangling
// mass) runs in the same CTA with coalesced accesses.  Replicas are mirrors
// (R19): not recomputed; the §2.4 merge (P@28309, mean P@28609) sets every
// copy.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "ktimer.h"
#include "sell.cuh"
#include "dist.h"

namespace gx {

struct PrState {
  double delta[3];   // L1 change of x_{t+1}, accumulated into [(t+1)%3]
  double dang[3];    // sum of x_t over dangling vertices, [t%3]
  double mass[3];    // sum of x_{t+1} over the vertices (owners), accumulated into [(t+1)%3]
  double scale;      // 1 / sum(x_t): lazy normalisation of iteration t's inputs (see k_pr_advance)
  unsigned iter;
  unsigned stop;     // 1 converged (delta < tol), 2 max_iters, 3 at the fp32-contrib noise floor
  double last_delta;
  double best_delta; // smallest delta so far (stagnation test)
  unsigned stall;    // iterations since best_delta last improved by >= 1 %
  unsigned merge_every;  // §2.4 cadence (gx_run_opts.merge_every)
  unsigned do_merge;     // iteration `iter` ends with a merge (set by k_pr_advance)
  unsigned force;        // the sweep reached its fixed point without a merge: merge next
  unsigned normalize;    // lazy normalisation on (off for the end-only merge, whose
                         // intermediate no-merge fixed point does not sum to 1)
  unsigned pb_next[3];   // blocked mapping: next sink bin of iteration t, [t%3]
};

struct PrArgs {
  // windowed SELL layout
  const uint32_t* slab;
  const uint32_t* slice_len;
  const uint64_t* slice_off;
  const int32_t* lane_row;
  const int32_t* heavy_row;
  const int64_t* win_slice;
  const int64_t* win_heavy;
  const uint32_t* crp;
  const int32_t* csrc;
  int64_t nwin;
  int64_t win_lo, win_hi;  // windows to sweep: [0, nwin)
  int64_t n_slots;         // rows of the layout (a rank's row count in the partitioned path)
  int64_t row0;            // global slot of layout row 0 (the rank's first row; 0 on one GPU)
  double* x;
  float* contrib[2];
  const uint32_t* D;
  const uint8_t* kind;   // null in exact mode
  const int32_t* gid;    // null without groups
  double* gnew;
  double base, damp, invN;
  PrState* st;
  int merge_bcast;       // 1: algorithm-aware merge (owner broadcast), else mean
  // TPV mapping (tpv.cu): lane-per-slot slabs of in-edges in schedule order
  const int32_t* tpv_lane_row;
  const uint32_t* tpv_len;
  const uint64_t* tpv_off;
  const uint32_t* tpv_slab;
  int64_t tpv_nslices;
};

// one atomic of each kind per CTA: L1 delta, dangling mass and total mass of
// the values this CTA wrote in iteration t
__device__ __forceinline__ void pr_flush(PrState* st, unsigned t, double my_delta, double my_dang, double my_mass,
                                         double* s_red) {
  double dsum = block_sum_f64(my_delta, s_red);
  __syncthreads();
  double gsum = block_sum_f64(my_dang, s_red);
  __syncthreads();
  double msum = block_sum_f64(my_mass, s_red);
  if (threadIdx.x == 0) {
    if (dsum != 0.0) atomicAdd(&st->delta[(t + 1) % 3], dsum);
    if (gsum != 0.0) atomicAdd(&st->dang[(t + 1) % 3], gsum);
    if (msum != 0.0) atomicAdd(&st->mass[(t + 1) % 3], msum);
  }
}

// contrib gather: read-only (.nc) in a Jacobi sweep; in the asynchronous
// schedule the buffer is written by the same sweep, so the load goes through
// L2 (.cg) and returns either the old or the new value of the source.
template <bool ASYNC>
__device__ __forceinline__ float ld_contrib(const float* p, uint64_t pol) {
  if (ASYNC) {
    float v;
    asm("ld.global.cg.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
  }
  return ld_keep_f32(p, pol);
}

template <bool SLOTS>
__device__ __forceinline__ void pr_finalize(const PrArgs& a, int64_t v, double y, double xo, uint32_t Dv, double addc,
                                            float* cout, double& my_delta, double& my_dang, bool merge_now, double sc,
                                            double& my_mass) {
  if (SLOTS) {
    if (a.kind[v] != OWNER) return;  // holes stay 0; replicas are set by the merge
  }
  double xn = addc + a.damp * sc * y;
  // a replicated owner hands its new value to the merge; in an iteration
  // without a merge (cadence N2) it updates its own copy only
  if (SLOTS && a.gid && merge_now) {
    int g = a.gid[v];
    if (g >= 0) {
      a.gnew[g] = xn;
      return;
    }
  }
  __stcs(a.x + v, xn);
  my_delta += fabs(xn - sc * xo);
  my_mass += xn;
  __stcs(cout + v, Dv ? (float)(xn / (double)Dv) : 0.0f);
  if (!Dv) my_dang += xn;
}

#ifndef GX_PR_CTA
#define GX_PR_CTA 256
#endif
constexpr int PR_CTA = GX_PR_CTA;
#ifndef GX_PR_U
#define GX_PR_U 8
#endif
#ifndef GX_PR_MINB
#define GX_PR_MINB 1
#endif
constexpr int PR_U = GX_PR_U;   // gathers in flight per lane

template <bool SLOTS, bool ASYNC>
__global__ void __launch_bounds__(PR_CTA, GX_PR_MINB) k_pr_sell(PrArgs a) {
  __shared__ double s_y[PRW];
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  const bool merge_now = st->do_merge != 0;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NWARP = PR_CTA / 32;
  for (int64_t w = a.win_lo + blockIdx.x; w < a.win_hi; w += gridDim.x) {
    const int64_t base = w * PRW;
    const int nrows = (int)min((int64_t)PRW, a.n_slots - base);
    for (int i = threadIdx.x; i < PRW; i += PR_CTA) s_y[i] = 0.0;
    __syncthreads();
    // light rows: lane-per-row over the SELL-32 slices of this window
    const int64_t s1 = a.win_slice[w + 1];
    for (int64_t sl = a.win_slice[w] + warp; sl < s1; sl += NWARP) {
      const uint32_t L = a.slice_len[sl];
      const uint32_t* p = a.slab + a.slice_off[sl] + lane;
      const int32_t row = a.lane_row[sl * 32 + lane];
      double acc = 0.0;
      uint32_t j = 0;
      for (; j + PR_U <= L; j += PR_U) {
        uint32_t e[PR_U];
#pragma unroll
        for (int u = 0; u < PR_U; u++) e[u] = ld_stream_u32(p + 32 * (j + u), pf);
        float v[PR_U];
#pragma unroll
        for (int u = 0; u < PR_U; u++) v[u] = e[u] != PR_SENT ? ld_contrib<ASYNC>(cin + e[u], pl) : 0.0f;
#pragma unroll
        for (int u = 0; u < PR_U; u++) acc += (double)v[u];
      }
      for (; j < L; j++) {
        uint32_t e = ld_stream_u32(p + 32 * j, pf);
        if (e != PR_SENT) acc += (double)ld_contrib<ASYNC>(cin + e, pl);
      }
      if (row >= 0) s_y[row - base] = acc;
    }
    // heavy rows: warp-per-row over the CSC
    const int64_t h1 = a.win_heavy[w + 1];
    for (int64_t h = a.win_heavy[w] + warp; h < h1; h += NWARP) {
      const int32_t r = a.heavy_row[h];
      const uint32_t e0 = a.crp[r], e1 = a.crp[r + 1];
      double acc = 0.0;
      for (uint32_t e = e0 + lane; e < e1; e += 32 * 4) {
        float v[4];
#pragma unroll
        for (int u = 0; u < 4; u++) {
          uint32_t ee = e + 32 * u;
          v[u] = ee < e1 ? ld_contrib<ASYNC>(cin + ld_stream_i32(a.csrc + ee, pf), pl) : 0.0f;
        }
#pragma unroll
        for (int u = 0; u < 4; u++) acc += (double)v[u];
      }
      acc = warp_sum_f64(acc);
      if (lane == 0) s_y[r - base] = acc;
    }
    __syncthreads();
    // fused update of the window's rows (coalesced x / D / contrib)
    for (int i0 = threadIdx.x; i0 < nrows; i0 += PR_CTA * 4) {
      double xo[4];
      uint32_t Dv[4];
#pragma unroll
      for (int u = 0; u < 4; u++) {
        int i = i0 + u * PR_CTA;
        xo[u] = i < nrows ? __ldcs(a.x + base + i) : 0.0;
        Dv[u] = i < nrows ? __ldcs(a.D + base + i) : 0u;
      }
#pragma unroll
      for (int u = 0; u < 4; u++) {
        int i = i0 + u * PR_CTA;
        if (i < nrows) pr_finalize<SLOTS>(a, base + i, s_y[i], xo[u], Dv[u], addc, cout, my_delta, my_dang, merge_now, sc,
                                              my_mass);
      }
    }
    __syncthreads();
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// v2 of the windowed SELL pull: (1) the window's x and D are bulk-copied
// (cp.async.bulk, one elected thread) into shared memory while the warps
// gather, so the fused update never waits on DRAM; (2) warps take work items
// -- heavy rows first, then the slices in their descending-length order --
// from a shared counter (longest-processing-time first), instead of a fixed
// round robin that leaves the warps with the longest slices as stragglers at
// the window barrier; (3) every row is written exactly once (lane_row and
// heavy_row partition the window), so s_y needs no zeroing pass.
template <bool SLOTS, bool ASYNC>
__global__ void __launch_bounds__(PR_CTA, GX_PR_MINB) k_pr_sell2(PrArgs a) {
  __shared__ double s_y[PRW];
  __shared__ __align__(128) double s_x[PRW];
  __shared__ __align__(128) uint32_t s_D[PRW];
  __shared__ double s_red[32];
  __shared__ __align__(8) uint64_t bar;
  __shared__ int s_next;
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  const bool merge_now = st->do_merge != 0;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const unsigned lane = lane_id();
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    mbar_fence_init();
    s_next = 0;
  }
  __syncthreads();
  unsigned phase = 0;
  for (int64_t w = a.win_lo + blockIdx.x; w < a.win_hi; w += gridDim.x) {
    const int64_t base = w * PRW;
    const int nrows = (int)min((int64_t)PRW, a.n_slots - base);
    const bool bulk = nrows == PRW;
    if (bulk && threadIdx.x == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_expect_tx(&bar, PRW * 12);
      tma_load_1d(s_x, a.x + a.row0 + base, PRW * 8, &bar, pf);
      tma_load_1d(s_D, a.D + a.row0 + base, PRW * 4, &bar, pf);
    }
    const int64_t s0 = a.win_slice[w], h0 = a.win_heavy[w];
    const int nh = (int)(a.win_heavy[w + 1] - h0), nit = nh + (int)(a.win_slice[w + 1] - s0);
    for (;;) {
      int it = 0;
      if (lane == 0) it = atomicAdd(&s_next, 1);
      it = __shfl_sync(FULL, it, 0);
      if (it >= nit) break;
      if (it < nh) {   // heavy row: warp-per-row over the CSC
        const int32_t r = a.heavy_row[h0 + it];
        const uint32_t e0 = a.crp[r], e1 = a.crp[r + 1];
        double acc = 0.0;
        for (uint32_t e = e0 + lane; e < e1; e += 32 * 4) {
          float v[4];
#pragma unroll
          for (int u = 0; u < 4; u++) {
            uint32_t ee = e + 32 * u;
            v[u] = ee < e1 ? ld_contrib<ASYNC>(cin + ld_stream_i32(a.csrc + ee, pf), pl) : 0.0f;
          }
#pragma unroll
          for (int u = 0; u < 4; u++) acc += (double)v[u];
        }
        acc = warp_sum_f64(acc);
        if (lane == 0) s_y[r - base] = acc;
        continue;
      }
      const int64_t sl = s0 + (it - nh);   // light slice: lane-per-row
      const uint32_t L = a.slice_len[sl];
      const uint32_t* p = a.slab + a.slice_off[sl] + lane;
      const int32_t row = a.lane_row[sl * 32 + lane];
      double acc = 0.0;
      uint32_t j = 0;
      for (; j + PR_U <= L; j += PR_U) {
        uint32_t e[PR_U];
#pragma unroll
        for (int u = 0; u < PR_U; u++) e[u] = ld_stream_u32(p + 32 * (j + u), pf);
        float v[PR_U];
#pragma unroll
        for (int u = 0; u < PR_U; u++) v[u] = e[u] != PR_SENT ? ld_contrib<ASYNC>(cin + e[u], pl) : 0.0f;
#pragma unroll
        for (int u = 0; u < PR_U; u++) acc += (double)v[u];
      }
      for (; j < L; j++) {
        uint32_t e = ld_stream_u32(p + 32 * j, pf);
        if (e != PR_SENT) acc += (double)ld_contrib<ASYNC>(cin + e, pl);
      }
      if (row >= 0) s_y[row - base] = acc;
    }
    if (bulk) mbar_wait(&bar, phase);
    phase ^= bulk ? 1u : 0u;
    __syncthreads();
    if (threadIdx.x == 0) s_next = 0;    // published by the barrier below
    for (int i = threadIdx.x; i < nrows; i += PR_CTA) {
      const double xo = bulk ? s_x[i] : __ldcs(a.x + a.row0 + base + i);
      const uint32_t Dv = bulk ? s_D[i] : __ldcs(a.D + a.row0 + base + i);
      pr_finalize<SLOTS>(a, a.row0 + base + i, s_y[i], xo, Dv, addc, cout, my_delta, my_dang, merge_now, sc,
                                              my_mass);
    }
    __syncthreads();
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// ---------------------------------------------------------------------------
// Propagation-blocked pull (GX_MAP_PB; PbLayout in gx_internal.h).  The sum
// of P@36969, y_v = sum_{u->v} x_u / D_u, is computed without any random
// global gather: every edge carries its term x_u/D_u in val[] (f32), laid out
// sink-bin major in (sink bin, source block) segments of PB_R-slot blocks.
// One CTA per SM claims sink bins in ascending order and, for bin b:
//   (1) streams the bin's contiguous range of val + 16-bit sink index with
//       16-byte loads and adds each term into a shared-memory accumulator of
//       its sink row (unsigned 64-bit fixed point, 2^-52 units, kept as two
//       32-bit words: exact, so the sum does not depend on the order); meanwhile the bin's
//       x / D rows are bulk-prefetched into L2;
//   (2) runs the PR update of the bin's rows (x, delta, dangling and total
//       mass as in pr_finalize) and keeps the new x/D of every row in shared
//       memory;
//   (3) scatters those terms along block b's out-edges: nb segments (one per
//       sink bin), each a 16-byte aligned run read with one 16-byte load of
//       source indices per lane and written as two float4 per lane.
// Bins later in the same sweep read the terms (3) just wrote, earlier bins
// read them next sweep: the asynchronous in-place schedule of the LB kernel
// (Theorem E3 fixes the limit; any mix of old and new terms is a valid
// chaotic-relaxation step).  Per edge and sweep: 4 + 2 bytes read in (1), 2
// read + 4 written in (3), all streaming -- 12 B against the 8 B of the
// gather pull, at HBM rate instead of the L1TEX random-sector rate.
// One CTA per SM (measured: two CTAs of half the rows, PB_R = 8192, are 18 %
// slower -- twice the segments, each half as long; a warp-specialised CTA
// running one bin's (1) beside the previous bin's (3) on separate warps was
// 5 % slower per sweep and needed 17 sweeps instead of 15, the scatter lagging
// one bin behind -- profiles/README.md "third session")
#ifndef GX_PB_THREADS
#define GX_PB_THREADS 1024
#endif
#ifndef GX_PB_CPS
#define GX_PB_CPS 1
#endif
constexpr int PB_THREADS = GX_PB_THREADS;
constexpr int PB_CTAS_PER_SM = GX_PB_CPS;
#ifndef GX_PB_PRODUCER
#define GX_PB_PRODUCER 1    // measured: 774 vs 813 us per sweep (RMAT-24)
#endif
#ifndef GX_PB_EPT
#define GX_PB_EPT 4
#endif
constexpr int PB_EPT = GX_PB_EPT;   // (1): terms per consumer thread per chunk (multiple of 4)
// (1): with a producer warp the last warp only issues the ring's bulk copies
// and the other 31 consume; else thread 0 issues between its own chunks
constexpr bool PB_PRODUCER = GX_PB_PRODUCER != 0;
constexpr int PB_CONSUMERS = PB_PRODUCER ? PB_THREADS - 32 : PB_THREADS;
constexpr int PB_CH = PB_EPT * PB_CONSUMERS;   // (1): elements per bulk-copied chunk
#ifndef GX_PB_NST
#define GX_PB_NST 4
#endif
constexpr int PB_NST = GX_PB_NST;  // (1): ring stages (NST - 1 chunks in flight while one is consumed)
constexpr size_t PB_STAGE = (size_t)PB_CH * 6;
#ifndef GX_PB_CPT
#define GX_PB_CPT 1
#endif
constexpr int PB_CPT = GX_PB_CPT;     // (1): ring chunks consumed per turn (4 terms each per thread)
#ifndef GX_PB_SEGU
#define GX_PB_SEGU 2    // measured: 1: 824, 2: 818, 4: 863, 8: 942 us per sweep (RMAT-24)
#endif
constexpr int PB_SEGU = GX_PB_SEGU;
#ifndef GX_PB_PFA
#define GX_PB_PFA 0    // measured: 0: 773, 4: 801, 8: 813, 16: 848, 32: 876 us per sweep (profiles/r1e)
#endif
constexpr int PB_PFA = GX_PB_PFA;     // (1): L2 prefetch distance of the bin stream, in chunks (0: off)   // (3): segments in flight per warp step (16-byte load each per lane)
// dynamic smem: acc_lo u32[R] (reused as the f32 terms s_c after the update)
// | 8 zero words (s_c[R..R+7], the padding entries' source) | acc_hi u32[R] | ring
constexpr size_t PB_RING_OFF = (size_t)PB_R * 8 + 32;
constexpr size_t PB_SMEM = PB_RING_OFF + PB_NST * PB_STAGE;

struct PbArgs {
  const uint32_t* q;
  const uint16_t* src_loc;
  const uint16_t* dst_loc;
  float* val;
  int64_t nb;
  int pack;   // (3) in packed steps (pb_scatter_packed): segments average fewer than PB_PACK_BELOW entries
};

__device__ __forceinline__ float4 ld_cg_f4(const float* p) {
  float4 v;
  asm volatile("ld.global.cg.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ void l2_prefetch_bulk(const void* p, uint32_t bytes) {
  if (bytes >= 16) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes & ~15u) : "memory");
}
// fixed-point accumulation with the one native shared-memory atomic (32-bit
// ATOMS.ADD; 64-bit and float adds compile to CAS loops): a term t >= 0 is
// v = rn(t * 2^F) (F = GX_PB_FIXBITS), kept as two 32-bit halves; the low half
// is added with a returning atomic and the high half (the term's own high bits
// plus the carry out of the low word) only when non-zero.  Exact and order
// independent.  F = 52 (quantum 2.2e-16, at most 1.1e-16 per edge, so the
// rounding of a whole sweep is below m * 2^-53 = 3e-8 in L1 at RMAT-24, well
// inside the 1e-6 tolerance) makes every term below 2^-20 -- all but a handful
// of RMAT terms x/D ~ 1e-8..1e-7 -- a single 32-bit value: measured, F = 56
// needed the second (high-word) atomic on 61 % of the terms (ncu source page,
// profiles/r2/pb_phase_split.txt).  The 64-bit accumulator holds sums up to
// 2^(64-F) = 4096 >= 1.
#ifndef GX_PB_FIXBITS
#define GX_PB_FIXBITS 52
#endif
#ifndef GX_PB_IFIX
#define GX_PB_IFIX 0    // measured slower: 713.5 (F2I.U64) vs 758 us per sweep (profiles/r1f/ifix_variants.txt)
#endif
constexpr float PB_FIX_SCALE = (float)(1ull << GX_PB_FIXBITS);
__device__ __forceinline__ unsigned long long pb_fix(float t) {
  // rn(t * 2^F) for a term 0 <= t <= 1 (the scaling is exact in f32, a subnormal t rounds to 0)
  if (!GX_PB_IFIX) return __float2ull_rn(t * PB_FIX_SCALE);
  const uint32_t b = __float_as_uint(t);
  const int e = (int)(b >> 23);   // biased exponent (t >= 0)
  const uint32_t m = (b & 0x7fffffu) | 0x800000u;
  const int sh = e - (150 - GX_PB_FIXBITS);   // t * 2^F = m * 2^(e - 127 - 23 + F)
  if (sh >= 0) return (unsigned long long)m << sh;
  const int r = -sh;
  if (e == 0 || r > 25) return 0ull;
  const uint32_t q = m >> r, rem = m & ((1u << r) - 1u), half = 1u << (r - 1);
  return q + ((rem > half || (rem == half && (q & 1u))) ? 1u : 0u);
}
__device__ __forceinline__ void pb_add4(uint32_t* lo, uint32_t* hi, uint2 r, float4 t4) {
  const uint32_t rr[4] = {r.x & 0xffffu, r.x >> 16, r.y & 0xffffu, r.y >> 16};
  const float tt[4] = {t4.x, t4.y, t4.z, t4.w};
  unsigned long long v[4];
  uint32_t old[4];
#pragma unroll
  for (int i = 0; i < 4; i++) v[i] = pb_fix(tt[i]);
  // the returning atomics are independent: issue them back to back
#pragma unroll
  for (int i = 0; i < 4; i++) old[i] = atomicAdd(&lo[rr[i]], (uint32_t)v[i]);
#pragma unroll
  for (int i = 0; i < 4; i++) {
    const uint32_t vl = (uint32_t)v[i];
    const uint32_t vh = (uint32_t)(v[i] >> 32) + (old[i] + vl < old[i] ? 1u : 0u);
    if (vh) atomicAdd(&hi[rr[i]], vh);
  }
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void pb_put8(float* dst, const float* s_c, uint4 w) {
  float4 o0, o1;
  o0.x = s_c[w.x & 0xffffu]; o0.y = s_c[w.x >> 16];
  o0.z = s_c[w.y & 0xffffu]; o0.w = s_c[w.y >> 16];
  o1.x = s_c[w.z & 0xffffu]; o1.y = s_c[w.z >> 16];
  o1.z = s_c[w.w & 0xffffu]; o1.w = s_c[w.w >> 16];
  __stcg(reinterpret_cast<float4*>(dst), o0);
  __stcg(reinterpret_cast<float4*>(dst) + 1, o1);
}

// the PR update of one row (pr_finalize) returning the row's next term x/D;
// false when the row is not recomputed here (hole, replica, or an owner that
// hands its value to the merge) -- its term is then the stored contrib
template <bool SLOTS>
__device__ __forceinline__ bool pb_update(const PrArgs& a, int64_t v, double y, double xo, uint32_t Dv, double addc,
                                          bool merge_now, double sc, double& my_delta, double& my_dang,
                                          double& my_mass, float& c) {
  if (SLOTS) {
    if (a.kind[v] != OWNER) return false;
  }
  const double xn = addc + a.damp * sc * y;
  if (SLOTS && a.gid && merge_now) {
    const int g = a.gid[v];
    if (g >= 0) {
      a.gnew[g] = xn;
      return false;
    }
  }
  __stcs(a.x + v, xn);
  my_delta += fabs(xn - sc * xo);
  my_mass += xn;
  c = Dv ? (float)(xn / (double)Dv) : 0.0f;
  // the stored contrib is read by the merge / local pass / merge carry only
  // (slot graphs); in exact mode the terms live in val[] alone
  if (SLOTS) __stcg(a.contrib[0] + v, c);
  if (!Dv) my_dang += xn;
  return true;
}

// (3): the terms s_c[0..PB_R) of one source block along its nb segments
// [r0[j], r1[j]) (16-byte aligned runs of 8-entry groups), 4 segments per warp
// step: one 16-byte load of source indices and two float4 stores per lane.
// lo0 / hi0 = the bounds of segment threadIdx.x (already loaded by the caller).
__device__ __forceinline__ void pb_scatter(const PbArgs& p, const float* s_c, const uint32_t* r0, const uint32_t* r1,
                                           uint32_t lo0, uint32_t hi0, uint64_t pf, unsigned warp = threadIdx.x >> 5,
                                           unsigned NW = PB_THREADS / 32, bool cached = true) {
  const unsigned lane = lane_id();
  const int64_t nb = p.nb;
  for (int64_t j0 = (int64_t)warp * 32; j0 < nb; j0 += 32 * NW) {
    const int64_t j = j0 + lane;
    const bool first = cached && j0 < 32 * NW;   // then segment j is thread j's (lo0, hi0)
    const uint32_t lo = first ? lo0 : j < nb ? __ldg(r0 + j) : 0u;
    const uint32_t hi = first ? hi0 : j < nb ? __ldg(r1 + j) : 0u;
    const int kn = (int)min((int64_t)32, nb - j0);
    for (int k = 0; k < kn; k += PB_SEGU) {
      uint32_t ee[PB_SEGU], hh[PB_SEGU];
      uint4 w[PB_SEGU];
#pragma unroll
      for (int u = 0; u < PB_SEGU; u++) {
        ee[u] = __shfl_sync(FULL, lo, k + u) + 8u * lane;
        hh[u] = __shfl_sync(FULL, hi, k + u);
        if (ee[u] < hh[u]) w[u] = ld_stream_v4(reinterpret_cast<const uint32_t*>(p.src_loc + ee[u]), pf);
      }
#pragma unroll
      for (int u = 0; u < PB_SEGU; u++) {
        if (ee[u] < hh[u]) pb_put8(p.val + ee[u], s_c, w[u]);
        for (uint32_t e = ee[u] + 256u; e < hh[u]; e += 256u)
          pb_put8(p.val + e, s_c, ld_stream_v4(reinterpret_cast<const uint32_t*>(p.src_loc + e), pf));
      }
    }
  }
}

// (3) with the source-index loads made asynchronous: each warp walks the same
// steps as pb_scatter (segment k of its 32-segment groups, 256 entries per
// step, one 16-byte group per lane) but copies a step's indices into its own
// slice of the (idle) bin-stream ring with cp.async and consumes them
// PB_SDEPTH steps later, so PB_SDEPTH x 512 B per warp are in flight without
// holding registers (pb_scatter's PB_SEGU register pipeline stops paying at 2).
// Each lane reads back only the 16 bytes it copied: no cross-lane hazard.
#ifndef GX_PB_SASYNC
#define GX_PB_SASYNC 1    // measured (RMAT-24, us per sweep): off 724.0, depth 3: 716.5, 4: 715.4, 5: 714.7 (profiles/r1f)
#endif
#ifndef GX_PB_SDEPTH
#define GX_PB_SDEPTH 4
#endif
constexpr int PB_SDEPTH = GX_PB_SDEPTH;
static_assert((size_t)PB_SDEPTH * 512 * (PB_THREADS / 32) <= (size_t)PB_NST * PB_STAGE, "scatter stages exceed the ring");
__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc, uint64_t pol) {
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc),
               "l"(pol)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
template <int DEPTH>
__device__ __forceinline__ void pb_scatter_async(const PbArgs& p, const float* s_c, const uint32_t* r0,
                                                 const uint32_t* r1, uint32_t lo0, uint32_t hi0, uint64_t pf,
                                                 uint4* stage /* this warp's DEPTH x 32 uint4 */) {
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = PB_THREADS / 32;
  const int64_t nb = p.nb;
  // warp-uniform step generator over segments j0 + k, k < kn, of groups j0 = warp*32 + i*32*NW
  int64_t j0 = (int64_t)warp * 32;
  uint32_t lo = lo0, hi = hi0;
  int kn = j0 < nb ? (int)min((int64_t)32, nb - j0) : 0;
  int k = 0;
  uint32_t eb = 0, hb = 0;
  if (kn) {
    eb = __shfl_sync(FULL, lo, 0);
    hb = __shfl_sync(FULL, hi, 0);
  }
  auto next = [&]() -> bool {   // (eb, hb): the next non-empty step
    while (kn) {
      if (eb < hb) return true;
      if (++k >= kn) {
        j0 += 32 * NW;
        k = 0;
        kn = j0 < nb ? (int)min((int64_t)32, nb - j0) : 0;
        if (!kn) return false;
        const int64_t j = j0 + lane;
        lo = j < nb ? __ldg(r0 + j) : 0u;
        hi = j < nb ? __ldg(r1 + j) : 0u;
      }
      eb = __shfl_sync(FULL, lo, k);
      hb = __shfl_sync(FULL, hi, k);
    }
    return false;
  };
  uint32_t pe[DEPTH];
  int pending = 0;
  bool more = true;
  auto refill = [&](int s) {
    pe[s] = 0xffffffffu;
    if (more) more = next();
    if (more) {
      const uint32_t e = eb + 8u * lane;
      if (e < hb) {
        pe[s] = e;
        cp_async16(stage + s * 32 + lane, p.src_loc + e, pf);
      }
      eb += 256u;
      pending++;
    }
    cp_async_commit();
  };
#pragma unroll
  for (int s = 0; s < DEPTH; s++) refill(s);
  while (pending) {
#pragma unroll
    for (int s = 0; s < DEPTH; s++) {
      cp_async_wait<DEPTH - 1>();
      if (pe[s] != 0xffffffffu) pb_put8(p.val + pe[s], s_c, stage[s * 32 + lane]);
      if (pending) pending--;   // stage s's step (issued in order) is consumed
      refill(s);
    }
  }
  cp_async_wait<0>();
}

// (3) with packed steps: a warp's 32 segments are treated as one run of
// 8-entry groups (a warp-wide inclusive scan of their group counts), and each
// step hands the next 32 groups to the 32 lanes whatever segment they fall in
// (a 5-round shuffle search of the scan), so short segments no longer leave
// most lanes of a step idle.  RMAT-24 averages 256 entries per segment, RMAT-26
// 64 (16.8M segments): one step per segment used 25 % of the lanes there.
// Loads asynchronous as in pb_scatter_async (cp.async into the warp's slice).
// Measured (profiles/r2/pb_pack_variants.txt, PageRank to 1e-9, per sweep):
// RMAT-26 (64 entries per segment) 3.72 -> 3.52 ms, RMAT-24 (256) 788 -> 783 us,
// RMAT-22 (1024) 214 -> 218 us: packed below 512 entries per segment
#ifndef GX_PB_PACK
#define GX_PB_PACK 1
#endif
#ifndef GX_PB_XPF
#define GX_PB_XPF 1   // (2)'s x / D rows prefetched into L2 at bin start
#endif
#ifndef GX_PB_PACK_BELOW
#define GX_PB_PACK_BELOW 512
#endif
template <int DEPTH>
__device__ __forceinline__ void pb_scatter_packed(const PbArgs& p, const float* s_c, const uint32_t* r0,
                                                  const uint32_t* r1, uint32_t lo0, uint32_t hi0, uint64_t pf,
                                                  uint4* stage /* this warp's DEPTH x 32 uint4 */) {
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = PB_THREADS / 32;
  const int64_t nb = p.nb;
  int64_t j0 = (int64_t)warp * 32;
  uint32_t lo = 0, incl = 0, G = 0, s0 = 0;
  // the segment holding group s0 (warp-uniform): its start, first group and end
  uint32_t ck = 0, clo = 0, cex = 0, cend = 0;
  auto locate = [&]() {
    ck = __ffs(__ballot_sync(FULL, incl > s0)) - 1;
    clo = __shfl_sync(FULL, lo, ck);
    cend = __shfl_sync(FULL, incl, ck);
    cex = __shfl_sync(FULL, incl, ck > 0 ? ck - 1 : 0);
    if (ck == 0) cex = 0u;
  };
  // the next 32-segment group holding any entry: lo = this lane's segment
  // start, incl = inclusive scan of the group counts, G = their total
  auto load_group = [&]() -> bool {
    while (j0 < nb) {
      const int64_t j = j0 + lane;
      uint32_t l = 0, h = 0;
      if (j < nb) {
        if (j0 < 32 * (int64_t)NW) {   // segment j = threadIdx.x: the caller's registers
          l = lo0;
          h = hi0;
        } else {
          l = __ldg(r0 + j);
          h = __ldg(r1 + j);
        }
      }
      lo = l;
      incl = warp_incl_scan_u32((h - l) >> 3);
      G = __shfl_sync(FULL, incl, 31);
      s0 = 0;
      if (G) {
        locate();
        return true;
      }
      j0 += 32 * NW;
    }
    return false;
  };
  bool more = load_group();
  uint32_t pe[DEPTH];
  int pending = 0;
  auto refill = [&](int s) {
    pe[s] = 0xffffffffu;
    if (more) {
      const uint32_t g = s0 + lane;
      uint32_t e;
      if (s0 + 32 <= cend) {   // the whole step inside one segment (long segments)
        e = clo + 8u * (g - cex);
      } else {                 // several segments: the segment of each lane's group by a shuffle search
        const uint32_t gq = min(g, G - 1u);
        int k = 0;
#pragma unroll
        for (int sft = 16; sft; sft >>= 1) {
          const uint32_t v = __shfl_sync(FULL, incl, k + sft - 1);
          if (v <= gq) k += sft;
        }
        uint32_t ex = __shfl_sync(FULL, incl, k > 0 ? k - 1 : 0);
        if (k == 0) ex = 0u;
        e = __shfl_sync(FULL, lo, k) + 8u * (gq - ex);
      }
      if (g < G) {
        pe[s] = e;
        cp_async16(stage + s * 32 + lane, p.src_loc + e, pf);
      }
      pending++;
      s0 += 32;
      if (s0 >= G) {
        j0 += 32 * NW;
        more = load_group();
      } else if (s0 >= cend) {
        locate();
      }
    }
    cp_async_commit();
  };
#pragma unroll
  for (int s = 0; s < DEPTH; s++) refill(s);
  while (pending) {
#pragma unroll
    for (int s = 0; s < DEPTH; s++) {
      cp_async_wait<DEPTH - 1>();
      if (pe[s] != 0xffffffffu) pb_put8(p.val + pe[s], s_c, stage[s * 32 + lane]);
      if (pending) pending--;   // stage s's step (issued in order) is consumed
      refill(s);
    }
  }
  cp_async_wait<0>();
}

// PACK: (3) in packed steps (one kernel per scatter: a run-time choice between
// the two inside one kernel measured an illegal-instruction fault on B200)
template <bool SLOTS, bool PACK>
__global__ void __launch_bounds__(PB_THREADS, PB_CTAS_PER_SM) k_pr_pb(PrArgs a, PbArgs p) {
  extern __shared__ __align__(16) unsigned char pb_smem[];
  uint32_t* acc_lo = reinterpret_cast<uint32_t*>(pb_smem);
  uint32_t* acc_hi = acc_lo + PB_R + 8;
  float* s_c = reinterpret_cast<float*>(acc_lo);   // terms, written over acc_lo by (2)
  unsigned char* ring = pb_smem + PB_RING_OFF;
  __shared__ double s_red[32];
  __shared__ int s_bin;
  __shared__ __align__(8) uint64_t full[PB_NST], empty[PB_NST];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  const bool merge_now = st->do_merge != 0;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const uint64_t pf = l2_evict_first();
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = PB_THREADS / 32;
  const int64_t nb = p.nb;
  const uint32_t* qend = p.q + nb * nb;
  const double inv_fix = 1.0 / (double)(1ull << GX_PB_FIXBITS);   // 2^-F
  if (threadIdx.x < 8) acc_lo[PB_R + threadIdx.x] = 0u;  // s_c[R..R+7] = 0.0f
  if (threadIdx.x == 0) {
    for (int i = 0; i < PB_NST; i++) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], PB_CONSUMERS / 32);
    }
    mbar_fence_init();
  }
  uint32_t g = 0;   // chunks this CTA has consumed (ring position), same in every thread
  // (1)'s producer (thread 0): chunk c of the range [e_lo, e_hi) into ring slot gc
  auto issue = [&](uint32_t gc, uint32_t e_lo, uint32_t e_hi, uint32_t c) {
    const uint32_t stg = gc % PB_NST;
    if (gc >= PB_NST) mbar_wait(&empty[stg], ((gc / PB_NST) - 1) & 1);
    const uint32_t e = e_lo + c * PB_CH, n = min((uint32_t)PB_CH, e_hi - e);
    unsigned char* dst = ring + stg * PB_STAGE;
    mbar_expect_tx(&full[stg], n * 6);
    tma_load_1d(dst, p.val + e, n * 4, &full[stg], pf);
    tma_load_1d(dst + PB_CH * 4, p.dst_loc + e, n * 2, &full[stg], pf);
  };
  for (;;) {
    if (threadIdx.x == 0) s_bin = (int)atomicAdd(&st->pb_next[t % 3], 1u);
    for (int i = threadIdx.x; i < PB_R / 4; i += PB_THREADS) {
      reinterpret_cast<uint4*>(acc_lo)[i] = make_uint4(0, 0, 0, 0);
      reinterpret_cast<uint4*>(acc_hi)[i] = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();
    const int64_t b = s_bin;
    if (b >= nb) break;
    const int64_t base = b * PB_R;
    const int nrows = (int)min((int64_t)PB_R, a.n_slots - base);
    const uint32_t* r0 = p.q + b * nb;   // block b's scatter segments: [r0[j], r1[j])
    const uint32_t* r1 = r0 + nb;
    // (1) the bin's in-edges: one contiguous range, bulk-copied chunk by chunk
    // into a PB_NST-stage shared-memory ring (one thread issues; each warp
    // releases a stage when it has added its part).  (Claiming the next bin
    // and starting its first chunks during (3) was measured 15 % slower: the
    // claiming warp's delay holds the whole CTA at the end of (3).)
    const uint32_t E0 = __ldg(p.q + b), E1 = __ldg(qend + b);
    const uint32_t nch = (E1 - E0 + PB_CH - 1) / PB_CH;
    if (threadIdx.x == 0) {
      if (!PB_PRODUCER)
        for (uint32_t c = 0; c < nch && c < PB_NST; c++) issue(g + c, E0, E1, c);
      // L2 prefetch for (2)
      if (GX_PB_XPF) {
        l2_prefetch_bulk(a.x + base, (uint32_t)nrows * 8u);
        l2_prefetch_bulk(a.D + base, (uint32_t)nrows * 4u);
      }
    }
    // (3)'s first PB_THREADS segment bounds stay in registers.  (An L2 prefetch
    // of every segment's source-index run here cost 6 % at RMAT-24 and 12 % at
    // RMAT-26 -- one bulk prefetch per segment, 16.8M per sweep there:
    // profiles/r2/pb_srcpf_variants.txt)
    uint32_t lo0 = 0, hi0 = 0;
    if (threadIdx.x < nb) {
      lo0 = __ldg(r0 + threadIdx.x);
      hi0 = __ldg(r1 + threadIdx.x);
    }
    if (PB_PRODUCER && threadIdx.x >= PB_CONSUMERS) {
      if (threadIdx.x == PB_CONSUMERS)
        for (uint32_t c = 0; c < nch; c++) {
          if (PB_PFA && c + PB_PFA < nch) {   // chunk c + PFA into L2 ahead of its bulk copy
            const uint32_t e = E0 + (c + PB_PFA) * PB_CH, n = min((uint32_t)PB_CH, E1 - e);
            l2_prefetch_bulk(p.val + e, n * 4u);
            l2_prefetch_bulk(p.dst_loc + e, n * 2u);
          }
          issue(g + c, E0, E1, c);
        }
    } else
    for (uint32_t c = 0; c < nch; c += PB_CPT) {
      constexpr int G4 = PB_EPT / 4;
      float4 tv[PB_CPT][G4];
      uint2 rv[PB_CPT][G4];
      bool ok[PB_CPT][G4];
#pragma unroll
      for (int q = 0; q < PB_CPT; q++) {
        const uint32_t cc = c + q, gc = g + cc, stg = gc % PB_NST;
#pragma unroll
        for (int h = 0; h < G4; h++) ok[q][h] = false;
        if (cc < nch) {
          const uint32_t n = min((uint32_t)PB_CH, E1 - (E0 + cc * PB_CH));
          mbar_wait(&full[stg], (gc / PB_NST) & 1);
          const unsigned char* src = ring + stg * PB_STAGE;
#pragma unroll
          for (int h = 0; h < G4; h++) {
            const uint32_t i = 4u * (threadIdx.x + h * PB_CONSUMERS);
            ok[q][h] = i < n;
            if (ok[q][h]) {
              tv[q][h] = *reinterpret_cast<const float4*>(src + 4 * i);
              rv[q][h] = *reinterpret_cast<const uint2*>(src + PB_CH * 4 + 2 * i);
            }
          }
        }
      }
#pragma unroll
      for (int q = 0; q < PB_CPT; q++)
#pragma unroll
        for (int h = 0; h < G4; h++)
          if (ok[q][h]) pb_add4(acc_lo, acc_hi, rv[q][h], tv[q][h]);
      __syncwarp();
#pragma unroll
      for (int q = 0; q < PB_CPT; q++) {
        const uint32_t cc = c + q, gc = g + cc;
        if (cc < nch) {
          if (lane == 0) mbar_arrive(&empty[gc % PB_NST]);
          if (!PB_PRODUCER && threadIdx.x == 0 && cc + PB_NST < nch) issue(gc + PB_NST, E0, E1, cc + PB_NST);
        }
      }
    }
    g += nch;
    __syncthreads();
    // (2) the PR update of the bin's rows
    for (int i0 = threadIdx.x; i0 < nrows; i0 += PB_THREADS * 4) {
      double xo[4];
      uint32_t Dv[4];
#pragma unroll
      for (int u = 0; u < 4; u++) {
        const int i = i0 + u * PB_THREADS;
        xo[u] = i < nrows ? __ldcs(a.x + base + i) : 0.0;
        Dv[u] = i < nrows ? __ldcs(a.D + base + i) : 0u;
      }
#pragma unroll
      for (int u = 0; u < 4; u++) {
        const int i = i0 + u * PB_THREADS;
        if (i < nrows) {
          const int64_t v = base + i;
          float c = 0.0f;
          const unsigned long long fx = ((unsigned long long)acc_hi[i] << 32) | acc_lo[i];
          if (!pb_update<SLOTS>(a, v, (double)fx * inv_fix, xo[u], Dv[u], addc, merge_now, sc, my_delta, my_dang,
                                my_mass, c))
            c = __ldcg(a.contrib[0] + v);
          s_c[i] = c;
        }
      }
    }
    __syncthreads();
    // (3) scatter the new terms along block b's segments
    if (GX_PB_SASYNC) {
      if (PACK)
        pb_scatter_packed<PB_SDEPTH>(p, s_c, r0, r1, lo0, hi0, pf, reinterpret_cast<uint4*>(ring) + warp * PB_SDEPTH * 32);
      else
        pb_scatter_async<PB_SDEPTH>(p, s_c, r0, r1, lo0, hi0, pf, reinterpret_cast<uint4*>(ring) + warp * PB_SDEPTH * 32);
      // the ring's next writes are the bulk copies (async proxy)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    } else
      pb_scatter(p, s_c, r0, r1, lo0, hi0, pf);
    __syncthreads();   // s_c (= acc_lo) is zeroed for the next bin
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// val[] <- the initial terms contrib_0[u] along every edge: (3) for every
// source block with s_c = contrib_0 of the block, each warp with a
// 2-deep cp.async staging slice after s_c
#ifndef GX_PB_INIT_SDEPTH
#define GX_PB_INIT_SDEPTH 2
#endif
constexpr int PB_INIT_SDEPTH = GX_PB_INIT_SDEPTH;
constexpr size_t PB_INIT_SMEM = (size_t)(PB_R + 8) * 4 + (GX_PB_SASYNC ? (size_t)(PB_THREADS / 32) * PB_INIT_SDEPTH * 512 : 0);
#ifndef GX_PB_INIT_MINB
#define GX_PB_INIT_MINB 1    // measured: 1 and 2 (32 registers, spill) tie (profiles/r1f/init_variants.txt)
#endif
template <bool PACK>
__global__ void __launch_bounds__(PB_THREADS, GX_PB_INIT_MINB) k_pb_init_val(PbArgs p, const float* __restrict__ contrib,
                                                               int64_t n_slots) {
  extern __shared__ __align__(16) float pb_init_s[];
  float* s_c = pb_init_s;   // PB_R + 8 floats
  const uint64_t pf = l2_evict_first();
  if (threadIdx.x < 8) s_c[PB_R + threadIdx.x] = 0.0f;
  for (int64_t b = blockIdx.x; b < p.nb; b += gridDim.x) {
    const int64_t base = b * PB_R;
    for (int i = threadIdx.x; i < PB_R; i += PB_THREADS) s_c[i] = base + i < n_slots ? contrib[base + i] : 0.0f;
    const uint32_t* r0 = p.q + b * p.nb;
    const uint32_t* r1 = r0 + p.nb;
    const uint32_t lo0 = threadIdx.x < p.nb ? r0[threadIdx.x] : 0u, hi0 = threadIdx.x < p.nb ? r1[threadIdx.x] : 0u;
    __syncthreads();
    if (GX_PB_SASYNC) {
      if (PACK)
        pb_scatter_packed<PB_INIT_SDEPTH>(p, s_c, r0, r1, lo0, hi0, pf,
                                          reinterpret_cast<uint4*>(s_c + PB_R + 8) + (threadIdx.x >> 5) * PB_INIT_SDEPTH * 32);
      else
        pb_scatter_async<PB_INIT_SDEPTH>(p, s_c, r0, r1, lo0, hi0, pf,
                                         reinterpret_cast<uint4*>(s_c + PB_R + 8) + (threadIdx.x >> 5) * PB_INIT_SDEPTH * 32);
    } else
      pb_scatter(p, s_c, r0, r1, lo0, hi0, pf);
    __syncthreads();
  }
}

// The paper's thread-per-vertex pull (tpv.cu): lane = slot of the schedule,
// each lane sums its own in-edges from the SELL-32 slab and finalises its
// slot; a warp lasts as long as its longest row (what §4 normalises).
template <bool SLOTS, bool ASYNC>
__global__ void __launch_bounds__(256) k_pr_tpv(PrArgs a) {
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  const bool merge_now = st->do_merge != 0;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const uint64_t pf = l2_evict_first(), pl = l2_evict_last();
  const unsigned lane = lane_id();
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t sl = gw; sl < a.tpv_nslices; sl += nw) {
    const int32_t row = a.tpv_lane_row[sl * 32 + lane];
    const uint32_t L = a.tpv_len[sl];
    const uint32_t* p = a.tpv_slab + a.tpv_off[sl] + lane;
    double acc = 0.0;
    uint32_t j = 0;
    for (; j + PR_U <= L; j += PR_U) {
      uint32_t e[PR_U];
#pragma unroll
      for (int u = 0; u < PR_U; u++) e[u] = row >= 0 ? ld_stream_u32(p + 32 * (j + u), pf) : PR_SENT;
      float v[PR_U];
#pragma unroll
      for (int u = 0; u < PR_U; u++) v[u] = e[u] != PR_SENT ? ld_contrib<ASYNC>(cin + e[u], pl) : 0.0f;
#pragma unroll
      for (int u = 0; u < PR_U; u++) acc += (double)v[u];
    }
    for (; j < L; j++) {
      uint32_t e = row >= 0 ? ld_stream_u32(p + 32 * j, pf) : PR_SENT;
      if (e != PR_SENT) acc += (double)ld_contrib<ASYNC>(cin + e, pl);
    }
    if (row >= 0) pr_finalize<SLOTS>(a, row, acc, __ldcs(a.x + row), __ldcs(a.D + row), addc, cout, my_delta, my_dang,
                                      merge_now, sc, my_mass);
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// 128 threads (4 warps) per tile.  Round 1 ran one thread per member and
// rescanned all of the tile's edges for every member in every local
// iteration (O(members x edges)); a hub member's CSC in-list was also walked by
// a single thread.  Now: warp-per-member external inflow, and the tile's edges
// regrouped by sink member in shared memory once per tile (a deterministic
// counting sort, one warp, __match_any_sync ranks), so a local iteration costs
// O(edges / threads).
constexpr int PRL_THREADS = 128;

// §3 shared-memory pass for PR (P@32188-32416; SURVEY A7 "PR store"): after
// the sweep, each subgraph tile iterates its members t times in shared
// memory, x_v <- (1-d)/N + d (ext_v + sum_{u in S, u->v} x_u / D_u + dang/N),
// where ext_v is the inflow from outside the tile (gathered from the CSC with
// the current contrib values).  Members that are replicated or not owners
// keep their sweep values and act as external sources.  The fixed point is
// unchanged (Theorem E3); delta grows by |x_loc - x_sweep| (an upper bound of
// the true change), dangling mass by the exact change.
// Dynamic shared memory: t_max_edges bytes (source member per in-edge).
template <bool SLOTS>
__global__ void __launch_bounds__(PRL_THREADS) k_pr_local(PrArgs a, const int32_t* __restrict__ tptr,
                                                  const int32_t* __restrict__ tmem, const int32_t* __restrict__ teptr,
                                                  const uint2* __restrict__ tedges, const int32_t* __restrict__ titers,
                                                  int64_t ntiles) {
  extern __shared__ uint8_t in_src[];
  __shared__ double xs[256], xn[256], ext[256], cs[256];
  __shared__ uint32_t Ds[256];
  __shared__ int32_t smem_id[256];
  __shared__ int in_ptr[257], cur[256];
  __shared__ uint8_t fixed[256];
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  constexpr unsigned NW = PRL_THREADS / 32;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int b0 = tptr[tile], nm = tptr[tile + 1] - b0;
    const int e0 = teptr[tile], ne = teptr[tile + 1] - e0;
    for (int i = threadIdx.x; i < nm; i += blockDim.x) {
      const int32_t v = tmem[b0 + i];
      bool fx = SLOTS && (a.kind[v] != OWNER || (a.gid && a.gid[v] >= 0));
      fixed[i] = fx;
      xs[i] = a.x[v];
      Ds[i] = a.D[v];
      smem_id[i] = v;
      cur[i] = 0;
    }
    __syncthreads();
    // in-degree of every member inside the tile
    for (int e = threadIdx.x; e < ne; e += blockDim.x) atomicAdd(&cur[(tedges[e0 + e].x >> 8) & 0xff], 1);
    __syncthreads();
    if (threadIdx.x == 0) {
      int acc = 0;
      for (int i = 0; i < nm; i++) {
        in_ptr[i] = acc;
        acc += cur[i];
        cur[i] = in_ptr[i];
      }
      in_ptr[nm] = acc;
    }
    __syncthreads();
    // edges regrouped by sink member, in tile-edge order within a sink (one
    // warp, 32 edges per step; lanes with the same sink ranked by match_any)
    if (warp == 0) {
      for (int c0 = 0; c0 < ne; c0 += 32) {
        const int e = c0 + (int)lane;
        const bool ok = e < ne;
        const uint32_t px = ok ? tedges[e0 + e].x : 0u;
        const int d = ok ? (int)((px >> 8) & 0xff) : 256 + (int)lane;
        const unsigned same = __match_any_sync(FULL, d);
        const int rank = __popc(same & lanemask_lt());
        if (ok) in_src[cur[d] + rank] = (uint8_t)(px & 0xff);
        __syncwarp();
        if (ok && rank == 0) cur[d] += __popc(same);
        __syncwarp();
      }
    }
    // external inflow, warp per member, from the CSC with the values the
    // contrib buffer holds now (sources outside the tile, or members that keep
    // their values); scaled like the sweep's inputs
    for (int i = warp; i < nm; i += NW) {
      double in = 0.0;
      if (!fixed[i]) {
        const int32_t v = smem_id[i];
        for (uint32_t e = a.crp[v] + lane; e < a.crp[v + 1]; e += 32) {
          const int32_t u = a.csrc[e];
          int lo = 0, hi = nm;   // members are sorted slot ids
          while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (smem_id[mid] < u) lo = mid + 1;
            else hi = mid;
          }
          const bool inside = lo < nm && smem_id[lo] == u && !fixed[lo];
          if (!inside) in += (double)cin[u];
        }
      }
      in = warp_sum_f64(in);
      if (lane == 0) ext[i] = sc * in;
    }
    __syncthreads();
    const int iters = titers[tile];
    for (int r = 0; r < iters; r++) {
      for (int i = threadIdx.x; i < nm; i += blockDim.x) cs[i] = (!fixed[i] && Ds[i]) ? xs[i] / (double)Ds[i] : 0.0;
      __syncthreads();
      for (int i = threadIdx.x; i < nm; i += blockDim.x) {
        if (fixed[i]) {
          xn[i] = xs[i];
          continue;
        }
        double in = ext[i];
        for (int k = in_ptr[i]; k < in_ptr[i + 1]; k++) in += cs[in_src[k]];
        xn[i] = addc + a.damp * in;
      }
      __syncthreads();
      for (int i = threadIdx.x; i < nm; i += blockDim.x) xs[i] = xn[i];
      __syncthreads();
    }
    for (int i = threadIdx.x; i < nm; i += blockDim.x) {
      if (fixed[i]) continue;
      const int32_t v = tmem[b0 + i];
      const double old = a.x[v];
      a.x[v] = xs[i];
      cout[v] = Ds[i] ? (float)(xs[i] / (double)Ds[i]) : 0.0f;
      my_delta += fabs(xs[i] - old);
      my_mass += xs[i] - old;
      if (!Ds[i]) my_dang += xs[i] - old;
    }
    __syncthreads();
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// Warp-per-tile version of k_pr_local (the default): each warp owns one tile
// at a time in its slice of dynamic shared memory (members, their values,
// sink-sorted local in-edges), so a 3-member tile costs a few warp
// instructions and no CTA barrier; the steps and the arithmetic are those of
// k_pr_local above.  Slice layout for TM members (multiple of 32) and TE
// local edges: double xs, xn, ext, cs [TM] | u32 Ds [TM] | i32 id [TM] |
// i32 in_ptr [TM + 1], cur [TM] | u8 fixed [TM] | u8 in_src [TE].
constexpr int PRLW_THREADS = 256;
__host__ __device__ inline size_t prlw_slice_bytes(int TM, int TE) {
  return (((size_t)TM * (4 * 8 + 4 + 4 + 4 + 4 + 1) + 4 + (size_t)TE) + 15) / 16 * 16;
}
template <bool SLOTS>
__global__ void __launch_bounds__(PRLW_THREADS) k_pr_local_warp(PrArgs a, const int32_t* __restrict__ tptr,
                                                              const int32_t* __restrict__ tmem,
                                                              const int32_t* __restrict__ teptr,
                                                              const uint2* __restrict__ tedges,
                                                              const int32_t* __restrict__ titers, int64_t ntiles,
                                                              int TM, int TE) {
  extern __shared__ __align__(16) unsigned char prlw_smem[];
  __shared__ double s_red[32];
  PrState* st = a.st;
  if (st->stop) return;
  const unsigned t = st->iter;
  const float* cin = a.contrib[t & 1];
  float* cout = a.contrib[(t + 1) & 1];
  const double sc = st->scale;
  const double addc = a.base + a.damp * sc * st->dang[t % 3] * a.invN;
  double my_delta = 0, my_dang = 0, my_mass = 0;
  const unsigned lane = lane_id(), warp = threadIdx.x >> 5;
  unsigned char* sl = prlw_smem + warp * prlw_slice_bytes(TM, TE);
  double* xs = reinterpret_cast<double*>(sl);
  double* xn = xs + TM;
  double* ext = xn + TM;
  double* cs = ext + TM;
  uint32_t* Ds = reinterpret_cast<uint32_t*>(cs + TM);
  int32_t* id = reinterpret_cast<int32_t*>(Ds + TM);
  int* in_ptr = id + TM;
  int* cur = in_ptr + TM + 1;
  uint8_t* fixed = reinterpret_cast<uint8_t*>(cur + TM);
  uint8_t* in_src = fixed + TM;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t tile = gw; tile < ntiles; tile += nw) {
    const int b0 = tptr[tile], nm = tptr[tile + 1] - b0;
    const int e0 = teptr[tile], ne = teptr[tile + 1] - e0;
    for (int i = lane; i < nm; i += 32) {
      const int32_t v = tmem[b0 + i];
      fixed[i] = SLOTS && (a.kind[v] != OWNER || (a.gid && a.gid[v] >= 0));
      xs[i] = a.x[v];
      Ds[i] = a.D[v];
      id[i] = v;
      cur[i] = 0;
    }
    __syncwarp();
    for (int e = lane; e < ne; e += 32) atomicAdd(&cur[(tedges[e0 + e].x >> 8) & 0xff], 1);
    __syncwarp();
    // exclusive scan of the in-degrees (nm <= 255: 8 steps of the warp scan)
    int carry = 0;
    for (int i0 = 0; i0 < nm; i0 += 32) {
      const int i = i0 + lane;
      const int c = i < nm ? cur[i] : 0;
      const int inc = (int)warp_incl_scan_u32((uint32_t)c);
      if (i < nm) {
        in_ptr[i] = carry + inc - c;
        cur[i] = carry + inc - c;
      }
      carry += __shfl_sync(FULL, inc, 31);
    }
    if (lane == 0) in_ptr[nm] = carry;
    __syncwarp();
    // edges regrouped by sink member, tile-edge order within a sink (match_any ranks)
    for (int c0 = 0; c0 < ne; c0 += 32) {
      const int e = c0 + (int)lane;
      const bool ok = e < ne;
      const uint32_t px = ok ? tedges[e0 + e].x : 0u;
      const int dd = ok ? (int)((px >> 8) & 0xff) : 256 + (int)lane;
      const unsigned same = __match_any_sync(FULL, dd);
      const int rank = __popc(same & lanemask_lt());
      if (ok) in_src[cur[dd] + rank] = (uint8_t)(px & 0xff);
      __syncwarp();
      if (ok && rank == 0) cur[dd] += __popc(same);
      __syncwarp();
    }
    // external inflow per member: the warp walks the member's CSC in-edges
    for (int i = 0; i < nm; i++) {
      double in = 0.0;
      if (!fixed[i]) {
        const int32_t v = id[i];
        for (uint32_t e = a.crp[v] + lane; e < a.crp[v + 1]; e += 32) {
          const int32_t u = a.csrc[e];
          int lo = 0, hi = nm;   // members are sorted slot ids
          while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (id[mid] < u) lo = mid + 1;
            else hi = mid;
          }
          const bool inside = lo < nm && id[lo] == u && !fixed[lo];
          if (!inside) in += (double)cin[u];
        }
      }
      in = warp_sum_f64(in);
      if (lane == 0) ext[i] = sc * in;
    }
    __syncwarp();
    const int iters = titers[tile];
    for (int r = 0; r < iters; r++) {
      for (int i = lane; i < nm; i += 32) cs[i] = (!fixed[i] && Ds[i]) ? xs[i] / (double)Ds[i] : 0.0;
      __syncwarp();
      for (int i = lane; i < nm; i += 32) {
        if (fixed[i]) {
          xn[i] = xs[i];
          continue;
        }
        double in = ext[i];
        for (int k = in_ptr[i]; k < in_ptr[i + 1]; k++) in += cs[in_src[k]];
        xn[i] = addc + a.damp * in;
      }
      __syncwarp();
      for (int i = lane; i < nm; i += 32) xs[i] = xn[i];
      __syncwarp();
    }
    for (int i = lane; i < nm; i += 32) {
      if (fixed[i]) continue;
      const int32_t v = id[i];
      const double old = a.x[v];
      a.x[v] = xs[i];
      cout[v] = Ds[i] ? (float)(xs[i] / (double)Ds[i]) : 0.0f;
      my_delta += fabs(xs[i] - old);
      my_mass += xs[i] - old;
      if (!Ds[i]) my_dang += xs[i] - old;
    }
    __syncwarp();
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
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
  if (!st->do_merge) {
    // iteration without a merge (cadence N2): replicas carry their values, and
    // under Jacobi their contributions must be carried into the next buffer
    const float* cin = a.contrib[t & 1];
    if (cin == cout) return;
    for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < ngroups; g += (int64_t)gridDim.x * blockDim.x)
      for (int i = gptr[g] + 1; i < gptr[g + 1]; i++) cout[gslots[i]] = cin[gslots[i]];
    return;
  }
  const double sc = st->scale;   // carried values are on the scale of x_t
  double my_delta = 0, my_dang = 0, my_mass = 0;
  for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < ngroups; g += (int64_t)gridDim.x * blockDim.x) {
    int b = gptr[g], e = gptr[g + 1];
    int32_t o = gslots[b];
    double s = a.gnew[g];
    for (int i = b + 1; i < e; i++) s += sc * a.x[gslots[i]];
    // GX_MERGE_MEAN: the paper's algorithm-agnostic mean (P@28609) over the
    // owner's new value and the replicas' carried values; the algorithm-aware
    // alternative (P@28421) for PR broadcasts the owner's new value (R54)
    double mean = a.merge_bcast ? a.gnew[g] : s / (double)(e - b);
    my_delta += fabs(mean - sc * a.x[o]);
    my_mass += mean;
    uint32_t Dv = a.D[o];
    float c = Dv ? (float)(mean / (double)Dv) : 0.0f;
    for (int i = b; i < e; i++) {
      a.x[gslots[i]] = mean;
      cout[gslots[i]] = c;
    }
    if (!Dv) my_dang += mean;
  }
  pr_flush(st, t, my_delta, my_dang, my_mass, s_red);
}

// loop state at iteration 0 (host copy: the merge cadence fields)
static void pr_state_init(PrState* dst, int merge_every, cudaStream_t s) {
  static PrState init;
  std::memset(&init, 0, sizeof(init));
  init.merge_every = (unsigned)merge_every;
  init.scale = 1.0;    // x0 = 1/N on every vertex sums to 1
  init.normalize = merge_every != 0 ? 1u : 0u;
  init.do_merge = merge_every == 1 ? 1u : 0u;   // iteration 0 merges iff (0 + 1) % c == 0
  // pageable source: the copy is staged before cudaMemcpyAsync returns
  CUDA_OK(cudaMemcpyAsync(dst, &init, sizeof(PrState), cudaMemcpyHostToDevice, s));
}

__global__ void k_pr_advance(PrState* st, double tol, int max_iters) {
  if (st->stop) return;
  unsigned t = st->iter;
  double dl = st->delta[(t + 1) % 3];
  st->last_delta = dl;
  // lazy normalisation: the next iteration scales its inputs by 1 / sum(x).
  // Jacobi conserves the mass (sum x = 1) by itself; the asynchronous schedule
  // and the §3 local pass do not, and a mass defect decays only at rate d per
  // iteration (R56).  The fixed point is unchanged (it has sum 1).
  const double ms = st->mass[(t + 1) % 3];
  st->scale = (st->normalize && ms > 0.0) ? 1.0 / ms : 1.0;
  st->delta[(t + 2) % 3] = 0.0;
  st->pb_next[(t + 2) % 3] = 0u;
  st->dang[(t + 2) % 3] = 0.0;
  st->mass[(t + 2) % 3] = 0.0;
  st->iter = t + 1;
  // contrib is stored in fp32: once the iterate reaches the fixed point of the
  // rounded map it may cycle at a delta floor ~1e-8..1e-9 (R55).
  // 32 iterations without a 1 % improvement below 1e-6 ends the loop there.
  if (t == 0 || dl < 0.99 * st->best_delta) {
    st->best_delta = dl;
    st->stall = 0;
  } else {
    st->stall++;
  }
  // merge cadence (P@28188 "after a certain number of iterations or at the
  // end of the overall computation"; gx_run_opts.merge_every = c):
  // c = 1 every iteration; c > 1 every c-th iteration, and a converged sweep
  // that did not merge merges in one more iteration before stopping; c = 0
  // only that final merge, after which the run ends.
  const unsigned c = st->merge_every;
  const bool merged = st->do_merge != 0;
  if (c == 0 && merged) {
    st->stop = 1;
    return;
  }
  const unsigned done = dl < tol ? 1u : (st->stall >= 32 && st->best_delta < 1e-6) ? 3u : 0u;
  if (done) {
    if (c == 1 || merged) st->stop = done;
    else st->force = 1;
  } else if ((int)(t + 1) >= max_iters) {
    st->stop = 2;
  }
  st->do_merge = (c == 1 || (c > 1 && (t + 2) % c == 0) || st->force) ? 1u : 0u;
  if (st->do_merge) st->force = 0;
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
    if (a.contrib[1] != a.contrib[0]) a.contrib[1][v] = 0.0f;
    if (k == OWNER && !Dv) my_dang += xv;
  }
  double gsum = block_sum_f64(my_dang, s_red);
  if (threadIdx.x == 0 && gsum != 0.0) atomicAdd(&a.st->dang[0], gsum);
}

void ensure_csc(gx_graph* g);  // devgraph.cu
void ensure_pb(gx_graph* g);   // devgraph.cu
void ensure_tpv(gx_graph* g);  // tpv.cu

RankLayouts& ensure_pr_ranks(gx_graph* g, int P, bool all);   // devgraph.cu

// the three scalars of iteration t (slot (t+1)%3: L1 delta, dangling mass,
// total mass) to / from the exchange buffer; a stopped loop leaves both alone
__global__ void k_pr_xch(PrState* st, double* xch, int unpack) {
  if (st->stop) return;
  const unsigned k = (st->iter + 1) % 3;
  if (!unpack) {
    xch[0] = st->delta[k];
    xch[1] = st->dang[k];
    xch[2] = st->mass[k];
  } else {
    st->delta[k] = xch[0];
    st->dang[k] = xch[1];
    st->mass[k] = xch[2];
  }
}

// 1-D partitioned PageRank (dist.h): rank p owns slot rows
// [lo_p, hi_p) (edge-balanced over in-edges) and stores only their in-CSC and
// windowed SELL (ensure_pr_ranks).  Per iteration:
//   sweep   k_pr_sell2 over the rank's windows, asynchronous in place inside
//           the rank (its own contrib slice is updated as it goes; the other
//           slices hold the previous exchange's values -- a chaotic
//           relaxation step, Theorem E3 keeps the fixed point)
//   reduce  ONE allreduce(sum) of [L1 delta, dangling, mass, group values]
//   gather  allgather(v) of the owned contrib slices (north_star: "allgathers
//           the rank vector for PageRank")
//   merge   §2.4 confluence, identical on every rank; advance (stop flag)
// No host synchronisation inside a batch of check_every iterations: every
// rank takes the same stop decision from the same reduced scalars, and the
// host reads the flag once per batch.
static void run_pagerank_dist(gx_graph* g, const gx_run_opts& o, gx_run_info& info, const PrArgs& a0, int P,
                              bool sim) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  const int64_t ns = d.n_slots, ng = d.n_groups;
  RankLayouts& RL = ensure_pr_ranks(g, P, sim);
  const std::vector<int64_t>& bounds = RL.bounds;
  const int nloc = sim ? P : 1;
  struct Rank {
    DBuf x, cb, xch, st;
    PrArgs a;
  };
  std::vector<Rank> R(nloc);
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  int64_t m_local = 0;
  for (int p = 0; p < nloc; p++) {
    Rank& K = R[p];
    const RankSlice& sl = RL.r[p];
    DBuf& x = p == 0 ? r.x : K.x;
    DBuf& cb = p == 0 ? r.contrib[0] : K.cb;
    DBuf& st = p == 0 ? r.pst : K.st;
    x.alloc(c, sizeof(double) * ns);
    cb.alloc(c, sizeof(float) * ns);
    st.alloc(c, sizeof(PrState));
    K.xch.alloc(c, sizeof(double) * (3 + ng));
    K.a = a0;
    K.a.x = x.as<double>();
    K.a.contrib[0] = K.a.contrib[1] = cb.as<float>();   // one buffer: in place inside the rank
    K.a.gnew = K.xch.as<double>() + 3;                  // group values ride in the fused allreduce
    K.a.st = st.as<PrState>();
    K.a.slab = sl.sell.slab.as<uint32_t>();
    K.a.slice_len = sl.sell.slice_len.as<uint32_t>();
    K.a.slice_off = sl.sell.slice_off.as<uint64_t>();
    K.a.lane_row = sl.sell.lane_row.as<int32_t>();
    K.a.heavy_row = sl.sell.heavy_row.as<int32_t>();
    K.a.win_slice = sl.sell.win_slice.as<int64_t>();
    K.a.win_heavy = sl.sell.win_heavy.as<int64_t>();
    K.a.crp = sl.crp.as<uint32_t>();
    K.a.csrc = sl.csrc.as<int32_t>();
    K.a.nwin = sl.sell.nwin;
    K.a.win_lo = 0;
    K.a.win_hi = sl.sell.nwin;
    K.a.n_slots = sl.hi - sl.lo;
    K.a.row0 = sl.lo;
    m_local += sl.m;
    pr_state_init(st.as<PrState>(), 1, s);
    if (d.identity) k_pr_init<false><<<grid_for(c, ns), 256, 0, s>>>(K.a, ns, 1.0 / (double)g->n);
    else k_pr_init<true><<<grid_for(c, ns), 256, 0, s>>>(K.a, ns, 1.0 / (double)g->n);
  }
  Exch X;
  X.c = c;
  X.P = P;
  X.sim = sim;
  int occ = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_sell2<true, true>, PR_CTA, 0));
  const int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((ng + 255) / 256, c->num_sms * 4));
  std::vector<void*> cbs, xs, xchs;
  for (int p = 0; p < nloc; p++) {
    cbs.push_back(R[p].a.contrib[0]);
    xs.push_back(R[p].a.x);
    xchs.push_back(R[p].xch.p);
  }
  const int batch = std::max(1, o.check_every);
  int launches = nloc, iters_enq = 0;
  PrState h;
  for (;;) {
    for (int it = 0; it < batch; it++, iters_enq++) {
      for (int p = 0; p < nloc; p++) {
        const PrArgs& A = R[p].a;
        if (ng) CUDA_OK(cudaMemsetAsync(A.gnew, 0, sizeof(double) * ng, s));
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(A.nwin, (int64_t)std::max(1, occ) * c->num_sms));
        if (d.identity) k_pr_sell2<false, true><<<grid, PR_CTA, 0, s>>>(A);
        else k_pr_sell2<true, true><<<grid, PR_CTA, 0, s>>>(A);
        k_pr_xch<<<1, 1, 0, s>>>(A.st, R[p].xch.as<double>(), 0);
        launches += 2;
      }
      X.allreduce(xchs, 3 + ng, Dt::F64, Op::SUM);   // delta, dangling, mass (+ group values): one collective
      for (int p = 0; p < nloc; p++) {
        k_pr_xch<<<1, 1, 0, s>>>(R[p].a.st, R[p].xch.as<double>(), 1);
        launches++;
      }
      X.allgatherv(cbs, bounds, Dt::F32);             // the owned contrib slices -> every rank
      for (int p = 0; p < nloc; p++) {
        if (ng) {
          k_pr_merge<<<grid_merge, 256, 0, s>>>(R[p].a, d.gptr.as<int32_t>(), d.gslots.as<int32_t>(), ng);
          launches++;
        }
        k_pr_advance<<<1, 1, 0, s>>>(R[p].a.st, o.tol, o.max_iters);
        launches++;
      }
    }
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaMemcpyAsync(&h, R[0].a.st, sizeof(PrState), cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    if (h.stop) break;
  }
  X.allgatherv(xs, bounds, Dt::F64);   // x: each slot from the rank that owns it
  CUDA_OK(cudaEventRecord(e1, s));
  CUDA_OK(cudaEventSynchronize(e1));
  float ms = 0;
  CUDA_OK(cudaEventElapsedTime(&ms, e0, e1));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  info.iterations = (int32_t)h.iter;
  info.converged = h.stop == 1 ? 1 : (h.stop == 3 ? 2 : 0);   // 2 = fp32 noise floor (R55)
  info.loop_ms = ms;
  info.last_delta = h.last_delta;
  // this rank's share of the work (the bench sums over ranks)
  info.edges_scanned = (int64_t)h.iter * (sim ? d.m_slots : m_local);
  info.vertices_active = (int64_t)h.iter * (sim ? ns : (RL.r[0].hi - RL.r[0].lo));
  info.bytes_model = 8 * info.edges_scanned + 32 * info.vertices_active;   // SURVEY §8(d) pull model
  info.kernel_launches = launches;
  info.mapping_used = GX_MAP_LB;
  r.have[GX_PAGERANK] = true;
}

void run_pagerank(gx_graph* g, const gx_run_opts& o, gx_run_info& info) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  RunState& r = g->rs;
  GX_CHECK_ARG(g->n > 0, "empty graph");
  int64_t ns = d.n_slots;
  // sweep mapping (one GPU); the blocked pull needs no CSC unless the §3 local
  // pass runs (it gathers the tiles' external inflow from the CSC)
  const int P_ranks = (c->world == 1 && o.sim_ranks > 1) ? o.sim_ranks : c->world;
  const bool async_ = o.pr_schedule == GX_PR_ASYNC && P_ranks == 1;
  const bool tiles = d.n_tiles && g->knobs.smem;
  int mapping = o.mapping;
  if (mapping == GX_MAP_AUTO) {
    // one CTA per SM claims sink bins: with fewer bins than SMs the last wave
    // leaves SMs idle.  Measured (profiles/r2): RMAT-22 (256 bins) PB 3.83 vs
    // LB 4.50 ms, RMAT-24 11.7 vs 17.2; with §3 tiles (C3 road) PB 176-395 vs
    // LB 380-895 and TPV 285-474 ms; §2 / §4 graphs PB best too (knobs tables)
    const bool pb_ok = async_ && (ns + PB_R - 1) / PB_R >= (int64_t)GX_PB_MIN_BINS_PER_SM * c->num_sms &&
                       !getenv("GX_NO_PB");
    mapping = pb_ok ? GX_MAP_PB : GX_MAP_LB;
  }
  if (mapping == GX_MAP_VNS) mapping = GX_MAP_TPV;   // a pull row is not split (graffix.h)
  if (P_ranks > 1 || mapping != GX_MAP_PB || tiles) resolve_pending(g);   // GX_ASYNC_UPLOAD: these layouts read {col, w}
  if (P_ranks == 1 && (mapping != GX_MAP_PB || tiles)) ensure_csc(g);   // partitioned: rank-local CSC only
  const bool sim_ = c->world == 1 && o.sim_ranks > 1;
  // the asynchronous schedule keeps ONE contrib buffer (read and written in
  // place by the sweep); Jacobi and the partitioned path need two
  const bool async = o.pr_schedule == GX_PR_ASYNC && c->world == 1 && !sim_;
  if (P_ranks == 1) {
    r.x.alloc(c, sizeof(double) * ns);
    r.contrib[0].alloc(c, sizeof(float) * ns);
    if (!async) r.contrib[1].alloc(c, sizeof(float) * ns);
    r.gnew.alloc(c, sizeof(double) * std::max<int64_t>(d.n_groups, 1));
    r.pst.alloc(c, sizeof(PrState));
  }
  PrArgs a;
  const SellLayout& PL = d.pr_sell;
  a.slab = PL.slab.as<uint32_t>();
  a.slice_len = PL.slice_len.as<uint32_t>();
  a.slice_off = PL.slice_off.as<uint64_t>();
  a.lane_row = PL.lane_row.as<int32_t>();
  a.heavy_row = PL.heavy_row.as<int32_t>();
  a.win_slice = PL.win_slice.as<int64_t>();
  a.win_heavy = PL.win_heavy.as<int64_t>();
  a.crp = d.crp.as<uint32_t>();
  a.csrc = d.csrc.as<int32_t>();
  a.nwin = PL.nwin;
  a.win_lo = 0;
  a.win_hi = PL.nwin;
  a.n_slots = ns;
  a.row0 = 0;
  a.x = r.x.as<double>();
  a.contrib[0] = r.contrib[0].as<float>();
  a.contrib[1] = async ? a.contrib[0] : r.contrib[1].as<float>();   // (the partitioned path sets its own)
  a.D = d.D.as<uint32_t>();
  a.kind = d.identity ? nullptr : d.kind.as<uint8_t>();
  a.gid = d.n_groups ? d.gid.as<int32_t>() : nullptr;
  a.gnew = r.gnew.as<double>();
  a.damp = o.damping;
  a.base = (1.0 - o.damping) / (double)g->n;
  a.invN = 1.0 / (double)g->n;
  a.st = r.pst.as<PrState>();
  a.merge_bcast = g->knobs.merge_op == GX_MERGE_MIN ? 1 : 0;
  const bool slots = !d.identity;
  {
    const bool sim = c->world == 1 && o.sim_ranks > 1;
    const int P = sim ? o.sim_ranks : c->world;
    if (P > 1) {
      GX_CHECK_ARG(P <= 8, "at most 8 ranks");
      GX_CHECK_ARG(o.mapping != GX_MAP_TPV && o.mapping != GX_MAP_PB && o.mapping != GX_MAP_VNS,
                   "the partitioned path uses the LB mapping");
      GX_CHECK_ARG(o.merge_every == 1 || !d.n_groups, "the partitioned path merges after every iteration");
      run_pagerank_dist(g, o, info, a, P, sim);
      return;
    }
  }
  GX_CHECK_ARG(mapping != GX_MAP_PB || async, "the blocked mapping runs the asynchronous schedule");
  PbArgs pb{};
  if (mapping == GX_MAP_PB) {
    ensure_pb(g);
    pb.q = d.pr_pb.q.as<uint32_t>();
    pb.src_loc = d.pr_pb.src_loc.as<uint16_t>();
    pb.dst_loc = d.pr_pb.dst_loc.as<uint16_t>();
    pb.val = d.pr_pb.val.as<float>();
    pb.nb = d.pr_pb.nb;
    pb.pack = (double)d.pr_pb.m_pad < (double)GX_PB_PACK_BELOW * (double)pb.nb * (double)pb.nb ? 1 : 0;
    if (const char* e = getenv("GX_PB_PACK_FORCE")) pb.pack = atoi(e) != 0;   // tests: either path on any graph
    // the opt-in is per device (context): set it on every run (cheap), not
    // once per process -- a second GPU in the same process needs it too
    CUDA_OK(cudaFuncSetAttribute(k_pr_pb<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_SMEM));
    CUDA_OK(cudaFuncSetAttribute(k_pr_pb<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_SMEM));
    CUDA_OK(cudaFuncSetAttribute(k_pr_pb<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_SMEM));
    CUDA_OK(cudaFuncSetAttribute(k_pr_pb<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_SMEM));
    CUDA_OK(cudaFuncSetAttribute(k_pb_init_val<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_INIT_SMEM));
    CUDA_OK(cudaFuncSetAttribute(k_pb_init_val<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)PB_INIT_SMEM));
  }
  if (mapping == GX_MAP_TPV) {
    ensure_tpv(g);
    a.tpv_lane_row = d.tpv_lane_row.as<int32_t>();
    a.tpv_len = d.tpv_in_len.as<uint32_t>();
    a.tpv_off = d.tpv_in_off.as<uint64_t>();
    a.tpv_slab = d.tpv_in_slab.as<uint32_t>();
    a.tpv_nslices = d.tpv_nslices;
  }

  if (tiles) {   // the warp-per-tile local pass may need more than 48 KB of dynamic shared memory
    CUDA_OK(cudaFuncSetAttribute(k_pr_local_warp<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    CUDA_OK(cudaFuncSetAttribute(k_pr_local_warp<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  }
  cudaEvent_t e0, e1;
  CUDA_OK(cudaEventCreate(&e0));
  CUDA_OK(cudaEventCreate(&e1));
  CUDA_OK(cudaEventRecord(e0, s));
  pr_state_init(a.st, d.n_groups ? o.merge_every : 1, s);
  int gi = grid_for(c, ns);
  if (slots) k_pr_init<true><<<gi, 256, 0, s>>>(a, ns, 1.0 / (double)g->n);
  else k_pr_init<false><<<gi, 256, 0, s>>>(a, ns, 1.0 / (double)g->n);
  const bool pack = GX_PB_PACK && pb.pack;
  if (mapping == GX_MAP_PB) {
    const int gi_pb = (int)std::min<int64_t>(pb.nb, c->num_sms * 2);
    if (pack) k_pb_init_val<true><<<gi_pb, PB_THREADS, PB_INIT_SMEM, s>>>(pb, a.contrib[0], ns);
    else k_pb_init_val<false><<<gi_pb, PB_THREADS, PB_INIT_SMEM, s>>>(pb, a.contrib[0], ns);
  }
  CUDA_OK(cudaGetLastError());
  int launches = mapping == GX_MAP_PB ? 2 : 1;
  const int grid_pb = (int)std::max<int64_t>(1, std::min<int64_t>(pb.nb, (int64_t)c->num_sms * PB_CTAS_PER_SM));

  // GX_PR_KERNEL=1 selects the round-1 kernel (A/B experiments)
  const bool v2 = !(getenv("GX_PR_KERNEL") && atoi(getenv("GX_PR_KERNEL")) == 1);
  int occ = 0;
  if (v2) CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_sell2<true, false>, PR_CTA, 0));
  else if (slots) CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_sell<true, false>, PR_CTA, 0));
  else CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pr_sell<false, false>, PR_CTA, 0));
  int grid = (int)std::max<int64_t>(1, std::min<int64_t>(PL.nwin, (int64_t)std::max(1, occ) * c->num_sms));
  int grid_merge = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_groups + 255) / 256, c->num_sms * 4));
  int occt = 0;
  CUDA_OK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occt, k_pr_tpv<true, false>, 256, 0));
  const int grid_tpv = std::max(1, occt) * c->num_sms;

  KTimer kt(o.profile != 0, s);
  auto one_iter = [&](int& nl) {
    kt.begin();
    if (mapping == GX_MAP_PB) {
      if (pack) {
        if (slots) k_pr_pb<true, true><<<grid_pb, PB_THREADS, PB_SMEM, s>>>(a, pb);
        else k_pr_pb<false, true><<<grid_pb, PB_THREADS, PB_SMEM, s>>>(a, pb);
      } else {
        if (slots) k_pr_pb<true, false><<<grid_pb, PB_THREADS, PB_SMEM, s>>>(a, pb);
        else k_pr_pb<false, false><<<grid_pb, PB_THREADS, PB_SMEM, s>>>(a, pb);
      }
    } else if (mapping == GX_MAP_TPV) {
      if (async) {
        if (slots) k_pr_tpv<true, true><<<grid_tpv, 256, 0, s>>>(a);
        else k_pr_tpv<false, true><<<grid_tpv, 256, 0, s>>>(a);
      } else {
        if (slots) k_pr_tpv<true, false><<<grid_tpv, 256, 0, s>>>(a);
        else k_pr_tpv<false, false><<<grid_tpv, 256, 0, s>>>(a);
      }
    } else {
      if (v2) {
        if (async) {
          if (slots) k_pr_sell2<true, true><<<grid, PR_CTA, 0, s>>>(a);
          else k_pr_sell2<false, true><<<grid, PR_CTA, 0, s>>>(a);
        } else {
          if (slots) k_pr_sell2<true, false><<<grid, PR_CTA, 0, s>>>(a);
          else k_pr_sell2<false, false><<<grid, PR_CTA, 0, s>>>(a);
        }
      } else if (async) {
        if (slots) k_pr_sell<true, true><<<grid, PR_CTA, 0, s>>>(a);
        else k_pr_sell<false, true><<<grid, PR_CTA, 0, s>>>(a);
      } else {
        if (slots) k_pr_sell<true, false><<<grid, PR_CTA, 0, s>>>(a);
        else k_pr_sell<false, false><<<grid, PR_CTA, 0, s>>>(a);
      }
    }
    kt.end();
    nl++;
    if (tiles) {
      // a warp per tile (k_pr_local_warp); GX_PR_LOCAL_CTA=1: the CTA-per-tile k_pr_local
      const int TM = (int)((std::max<int64_t>(d.t_max_members, 1) + 31) / 32 * 32);
      const int TE = (int)std::max<int64_t>(d.t_max_edges, 16);
      const size_t wsm = prlw_slice_bytes(TM, TE) * (PRLW_THREADS / 32);
      if (!getenv("GX_PR_LOCAL_CTA") && wsm <= 200 * 1024) {
        const int grid_lw = (int)std::max<int64_t>(1, std::min<int64_t>((d.n_tiles + 7) / 8, (int64_t)c->num_sms * 8));
        if (slots)
          k_pr_local_warp<true><<<grid_lw, PRLW_THREADS, wsm, s>>>(a, d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(),
                                                                  d.t_eptr.as<int32_t>(), d.t_edges.as<uint2>(),
                                                                  d.t_iters.as<int32_t>(), d.n_tiles, TM, TE);
        else
          k_pr_local_warp<false><<<grid_lw, PRLW_THREADS, wsm, s>>>(a, d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(),
                                                                   d.t_eptr.as<int32_t>(), d.t_edges.as<uint2>(),
                                                                   d.t_iters.as<int32_t>(), d.n_tiles, TM, TE);
        nl++;
      } else {
      const int grid_local = (int)std::max<int64_t>(1, std::min<int64_t>(d.n_tiles, (int64_t)c->num_sms * 16));
      const size_t prl_smem = (size_t)std::max<int64_t>(d.t_max_edges, 16);
      if (slots)
        k_pr_local<true><<<grid_local, PRL_THREADS, prl_smem, s>>>(a, d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(),
                                                    d.t_eptr.as<int32_t>(), d.t_edges.as<uint2>(), d.t_iters.as<int32_t>(),
                                                    d.n_tiles);
      else
        k_pr_local<false><<<grid_local, PRL_THREADS, prl_smem, s>>>(a, d.t_ptr.as<int32_t>(), d.t_members.as<int32_t>(),
                                                     d.t_eptr.as<int32_t>(), d.t_edges.as<uint2>(),
                                                     d.t_iters.as<int32_t>(), d.n_tiles);
      nl++;
      }
    }
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
  info.converged = h.stop == 1 ? 1 : (h.stop == 3 ? 2 : 0);   // 2 = fp32 noise floor (R55)
  info.loop_ms = ms;
  info.last_delta = h.last_delta;
  info.edges_scanned = (int64_t)h.iter * d.m_slots;
  info.vertices_active = (int64_t)h.iter * ns;
  // bytes model (SURVEY.md §8(d) pull model): 8 B per in-edge (source id 4 +
  // contrib gather 4) and 32 B per slot (row_ptr 8 + x read 8 + x write 8 +
  // contrib write 4 + D 4)
  info.bytes_model = (int64_t)h.iter * (8 * d.m_slots + 32 * ns);
  info.kernel_launches = launches;
  info.sweep_launches = kt.launches();
  info.sweep_ms = kt.total_ms();
  // the bytes the sweep kernel's own encoding moves: the blocked mapping
  // (k_pr_pb) streams 12 B per edge (val 4 + sink index 2 read, source index 2
  // read + val 4 written) and 28 B per slot (x r/w 16, D 4, contrib write 4,
  // segment offsets ~4) instead of the pull's 8 B gather per edge
  info.sweep_bytes = mapping == GX_MAP_PB ? (int64_t)h.iter * (12 * d.m_slots + 28 * ns) : info.bytes_model;
  info.mapping_used = mapping;
  r.have[GX_PAGERANK] = true;
}

}  // namespace gx
