// sssp_common.cuh -- frontier state shared by the SSSP sweep kernels.
#pragma once
#include <cstdint>

namespace gx {

constexpr uint32_t HEAVY_DEG = 256;  // out-degree above which a slot is split into static chunks
constexpr uint32_t HCHUNK = 1024;    // edges per heavy chunk

// Device-side loop state.  The frontier is a 1-bit-per-slot bitmap,
// triple-buffered by iteration (bm[t%3] current, bm[(t+1)%3] next,
// bm[(t+2)%3] being cleared), so one iteration needs no host round trip.
struct SsspState {
  unsigned int iter;            // current iteration t
  unsigned int stop;            // 0 running, 1 converged (empty frontier), 2 max_iters
  unsigned int active[3];       // frontier slots processed in iteration t
  unsigned int pushed[3];       // next-frontier bits set in iteration t (0 => the next frontier is empty);
                                // contiguous with active[] so one allreduce sums both (dist.h)
  unsigned int tau;             // near-far threshold: relaxations to dist >= tau go to the far pile
  unsigned int delta;           // bucket width (0 = plain Bellman-Ford frontier)
  unsigned int far_min;         // upper bound of the smallest distance in the far pile (INF = empty)
  unsigned int split;           // 1: the near frontier drained, refill it from the far pile
  unsigned int raised;          // merges that raised a copy (diagnostic)
  unsigned long long edges;     // edges relaxed, all iterations
  unsigned long long act_total; // frontier entries, all iterations
  unsigned int merge_every;     // §2.4 cadence c (gx_run_opts.merge_every; 1 when there are no replicas)
  unsigned int do_merge;        // iteration `iter` ends with a merge
  unsigned int final_merge;     // c = 0: this iteration's merge ends the run
  unsigned int far3[3];         // persistent loop: far-pile minimum pushed in iteration t, [t%3]
  unsigned int tiles_n[3];      // §3 tiles touched in iteration t (list length), [t%3]
  unsigned long long refill_deg[3];  // slots a near-far refill moved into frontier t, [t%3]
  unsigned int dense_bin;       // blocked dense relaxation: next sink bin to claim
  unsigned int wmul;            // near-far window = delta * wmul (doubles after small refills; 0 reads as 1)
  // frontier windows (persistent LB loop, win_on): the bits of frontier k
  // (bm[k%3]) lie only in words [wlo[k%6], whi[k%6]] (wlo > whi: empty), the
  // far pile's bits in [flo[e&1], fhi[e&1]] for refill epoch e; the scan, the
  // clear of the recycled bitmap and the refill touch only those words.  Six
  // slots, not three: the lead empties frontier k's slot in the decision of
  // iteration k+1 (no barrier follows it), and that slot's next pushes come
  // three grid barriers later (frontier k+6), never racing the reset
  unsigned int win_on;
  unsigned int wlo[6], whi[6];
  unsigned int flo[2], fhi[2];
  unsigned int epoch;
  unsigned int tau_prev;        // far-by-scan refills: the bucket bound before the last raise of tau
};

struct SsspAux {
  uint32_t* bm[3];              // frontier bitmaps
  uint32_t* far;                // near-far: slots waiting for a later bucket
  const uint32_t* heavy;        // bitmap: out-degree > HEAVY_DEG
  int64_t nwords;
  const int32_t* hc_row;        // static heavy chunk list: row
  const uint32_t* hc_start;     //                          first edge
  int64_t nhc;
  // packed out-edges (null: use the uint2 {dst, w} array): dst << wbits | w in
  // one u32 when n' <= 2^(32 - wbits) -- 4 bytes per relaxed edge instead of 8
  const uint32_t* adjp;
  uint32_t wbits;
  // light / heavy edge split (delta-stepping's edge classes; null: off):
  // row u's edges [rp[u], lend[u]) have w < delta, [lend[u], rp[u+1]) w >= delta.
  // A light pass relaxes the light edges of the frontier and records it in
  // pend[p]; a heavy pass relaxes the heavy edges of pend[p] once the bucket
  // drained (a heavy edge from the bucket cannot land below tau, sssp.cu)
  const uint32_t* lend;
  uint32_t* pend[2];
};
// du + w, saturated at 2^32-2 (reading R51): every sum that wraps or lands on
// INF becomes INF-1, which k_sat_check reports as an overflow after the run
__device__ __forceinline__ uint32_t sat_add(uint32_t du, uint32_t w) {
  const uint32_t nd = du + w;
  return (nd < du || nd == 0xFFFFFFFFu) ? 0xFFFFFFFEu : nd;
}

// the out-edge e as {dst, w}.  GX_SSSP_EDGE_VOLATILE=1 pins the program order
// (the LB sweep's next-round edge loads before this round's dist gathers); the
// compiler otherwise sinks them to their use (ncu source page, profiles/r2),
// but pinned they measured slower: RMAT-24 4.60 (free) vs 4.94-5.02 ms
// (SU 2-4, profiles/r2/sssp_edge_volatile_variants.txt)
#ifndef GX_SSSP_EDGE_VOLATILE
#define GX_SSSP_EDGE_VOLATILE 0
#endif
#if GX_SSSP_EDGE_VOLATILE
#define GX_EDGE_ASM asm volatile
#else
#define GX_EDGE_ASM asm
#endif
__device__ __forceinline__ uint32_t ld_edge_raw(const uint32_t* p, uint64_t pol) {
  uint32_t v;
  GX_EDGE_ASM("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint2 ld_edge(const uint2* __restrict__ adj, const SsspAux& ax, uint32_t e, uint64_t pol) {
  if (ax.adjp) {
    const uint32_t v = ld_edge_raw(ax.adjp + e, pol);
    return make_uint2(v >> ax.wbits, v & ((1u << ax.wbits) - 1u));
  }
  uint2 v;
  GX_EDGE_ASM("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;" : "=r"(v.x), "=r"(v.y)
              : "l"(adj + e), "l"(pol));
  return v;
}

}  // namespace gx
