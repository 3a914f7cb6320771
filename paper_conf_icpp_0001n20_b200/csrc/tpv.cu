// tpv.cu -- layout of the paper's vertex-centric mapping (PAPER.md P@15381:
// "a thread is assigned to a vertex"; a warp processes consecutive vertices,
// P@24189).  Lane l of warp w owns slot sched[32w + l]: the §4 warp schedule
// when degree normalisation is on (P@33432), else slot order -- which, after
// the §2 renumbering, puts the children of one parent chunk into one warp.
// Edges are stored as SELL-32 slabs in that lane order, so the j-th edges of
// a warp's 32 slots are one coalesced load; the slab is padded to the longest
// row of the warp, which is exactly the divergence §4 reduces.  The sweeps
// themselves are k_sssp_tpv (sssp.cu) and k_pr_tpv (pagerank.cu).
#include <algorithm>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "sell.cuh"

namespace gx {

void ensure_csc(gx_graph* g);  // devgraph.cu

void ensure_tpv(gx_graph* g) {
  DevGraph& d = g->dg;
  if (d.tpv_ready) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  ensure_csc(g);
  const int64_t ns = d.n_slots;
  // lane order: §4 schedule if present, else every slot in slot order
  std::vector<int32_t> lanes;
  if (g->transformed && !g->sg.sched.empty()) lanes = g->sg.sched;
  else {
    lanes.resize(ns);
    for (int64_t i = 0; i < ns; i++) lanes[i] = (int32_t)i;
  }
  const int64_t nsl = ((int64_t)lanes.size() + 31) / 32;
  lanes.resize(nsl * 32 + 32, -1);
  d.tpv_nslices = nsl;
  d.tpv_lane_row.alloc(c, sizeof(int32_t) * lanes.size());
  CUDA_OK(cudaMemcpyAsync(d.tpv_lane_row.p, lanes.data(), sizeof(int32_t) * lanes.size(), cudaMemcpyHostToDevice, s));
  d.tpv_out_slab_len = build_sell<uint2>(c, d.rp.as<uint32_t>(), d.adj.as<uint2>(), d.tpv_lane_row.as<int32_t>(), nsl,
                                         make_uint2(0xFFFFFFFFu, 0u), d.tpv_out_len, d.tpv_out_off, d.tpv_out_slab);
  d.tpv_in_slab_len = build_sell<uint32_t>(c, d.crp.as<uint32_t>(), reinterpret_cast<const uint32_t*>(d.csrc.p),
                                           d.tpv_lane_row.as<int32_t>(), nsl, PR_SENT, d.tpv_in_len, d.tpv_in_off,
                                           d.tpv_in_slab);
  CUDA_OK(cudaStreamSynchronize(s));
  d.tpv_ready = true;
}

}  // namespace gx
