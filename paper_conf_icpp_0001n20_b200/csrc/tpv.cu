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
void launch_vns_gather(Ctx* c, const uint32_t* vr, const uint32_t* crp, const uint2* adj, int64_t nv, uint2* out);

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

// Virtual node splitting (Tigr, the engine of the paper's second workload):
// virtual node = a run of at most K consecutive out-edges of one slot, so the
// virtual rows are sub-ranges of the slot CSR and the slab builder reads them
// straight from `adj` through a virtual row pointer.  Virtual nodes follow the
// TPV lane order (the §4 schedule or slot order, i.e. the §2 layout).
void ensure_vns(gx_graph* g) {
  DevGraph& d = g->dg;
  int K = 8;
  if (const char* e = getenv("GX_VNS_K")) K = std::max(1, std::min(atoi(e), 1 << 20));
  if (d.vns_ready && d.vns_k == K) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  const int64_t ns = d.n_slots;
  std::vector<uint32_t> rp(ns + 1);
  CUDA_OK(cudaMemcpyAsync(rp.data(), d.rp.p, sizeof(uint32_t) * (ns + 1), cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  std::vector<int32_t> order;
  if (g->transformed && !g->sg.sched.empty()) order = g->sg.sched;
  else {
    order.resize(ns);
    for (int64_t i = 0; i < ns; i++) order[i] = (int32_t)i;
  }
  std::vector<uint32_t> vrp;     // virtual row pointers into adj: [2v] start, [2v+1] end (pairs)
  std::vector<int32_t> lslot;
  for (int32_t sl : order) {
    const uint32_t a = rp[sl], b = rp[sl + 1];
    for (uint32_t e = a; e < b; e += (uint32_t)K) {
      vrp.push_back(e);
      vrp.push_back(std::min(b, e + (uint32_t)K));
      lslot.push_back(sl);
    }
  }
  const int64_t nv = (int64_t)lslot.size();
  const int64_t nsl = (nv + 31) / 32;
  // the slab builder takes a CSR row pointer: virtual rows are not contiguous
  // in adj order (lane order may differ from slot order), so give it a
  // gathered copy of the edges in virtual-row order with a compact pointer
  std::vector<uint32_t> crp(nv + 1, 0);
  for (int64_t v = 0; v < nv; v++) crp[v + 1] = crp[v] + (vrp[2 * v + 1] - vrp[2 * v]);
  std::vector<int32_t> lanes(nsl * 32 + 32, -1), lslot_p(nsl * 32 + 32, -1);
  for (int64_t v = 0; v < nv; v++) {
    lanes[v] = (int32_t)v;
    lslot_p[v] = lslot[v];
  }
  DBuf dvr, dcrp, dgat, dlanes;
  dvr.alloc(c, sizeof(uint32_t) * std::max<int64_t>(2 * nv, 2));
  dcrp.alloc(c, sizeof(uint32_t) * (nv + 1));
  dgat.alloc(c, sizeof(uint2) * std::max<int64_t>(crp[nv], 1));
  dlanes.alloc(c, sizeof(int32_t) * lanes.size());
  if (nv) CUDA_OK(cudaMemcpyAsync(dvr.p, vrp.data(), sizeof(uint32_t) * 2 * nv, cudaMemcpyHostToDevice, s));
  CUDA_OK(cudaMemcpyAsync(dcrp.p, crp.data(), sizeof(uint32_t) * (nv + 1), cudaMemcpyHostToDevice, s));
  CUDA_OK(cudaMemcpyAsync(dlanes.p, lanes.data(), sizeof(int32_t) * lanes.size(), cudaMemcpyHostToDevice, s));
  if (nv) launch_vns_gather(c, dvr.as<uint32_t>(), dcrp.as<uint32_t>(), d.adj.as<uint2>(), nv, dgat.as<uint2>());
  d.vns_lane_slot.alloc(c, sizeof(int32_t) * lslot_p.size());
  CUDA_OK(cudaMemcpyAsync(d.vns_lane_slot.p, lslot_p.data(), sizeof(int32_t) * lslot_p.size(), cudaMemcpyHostToDevice,
                          s));
  build_sell<uint2>(c, dcrp.as<uint32_t>(), dgat.as<uint2>(), dlanes.as<int32_t>(), nsl, make_uint2(0xFFFFFFFFu, 0u),
                    d.vns_len, d.vns_off, d.vns_slab);
  CUDA_OK(cudaStreamSynchronize(s));
  d.vns_nslices = nsl;
  d.vns_nv = nv;
  d.vns_k = K;
  d.vns_ready = true;
}

__global__ void k_vns_gather(const uint32_t* __restrict__ vr, const uint32_t* __restrict__ crp,
                             const uint2* __restrict__ adj, int64_t nv, uint2* __restrict__ out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < nv; v += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t a = vr[2 * v], b = vr[2 * v + 1], o = crp[v];
    for (uint32_t e = a; e < b; e++) out[o + (e - a)] = adj[e];
  }
}
void launch_vns_gather(Ctx* c, const uint32_t* vr, const uint32_t* crp, const uint2* adj, int64_t nv, uint2* out) {
  k_vns_gather<<<grid_for(c, nv), 256, 0, c->stream>>>(vr, crp, adj, nv, out);
  CUDA_OK(cudaGetLastError());
}

}  // namespace gx
