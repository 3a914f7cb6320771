// devgraph.cu -- device layouts of the (transformed) slot graph.
//
//  * out-CSR  rp u32[n'+1], adj uint2{col, w}[m']: one 8-byte coalesced load
//    per relaxed edge (SSSP push, BC, SCC forward);
//  * in-CSC   crp u32[n'+1], csrc i32[m'] rows sorted by source slot (built on
//    the device with a radix sort of (dst, src) keys): PR pull, SCC backward;
//  * PR merge-path tiles over (rows + in-edges) and the rows spanning tiles;
//  * D u32[n'] = logical out-degree of the slot's vertex (PR divisor; for a
//    replicated vertex the SUM over its copies);
//  * confluence groups (owner first) with the owner's in-edges for the
//    SSSP re-pull after a merge.
#include <cub/cub.cuh>

#include <algorithm>
#include <numeric>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "sell.cuh"
#include "dist.h"

namespace gx {

// ------------------------------------------------------------------ kernels
__global__ void k_rp64_to_u32(const int64_t* __restrict__ in, uint32_t* __restrict__ out, int64_t n1) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n1; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (uint32_t)in[i];
}

__global__ void k_interleave(const int32_t* __restrict__ col, const uint32_t* __restrict__ w,
                             uint2* __restrict__ adj, int64_t m) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
    adj[e] = make_uint2((uint32_t)col[e], w ? w[e] : 1u);
}

__global__ void k_outdeg(const uint32_t* __restrict__ rp, uint32_t* __restrict__ D, int64_t n) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    D[v] = rp[v + 1] - rp[v];
}

__global__ void k_validate(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                           const uint32_t* __restrict__ w, int64_t n, int64_t m,
                           unsigned int* __restrict__ err) {
  int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
  for (int64_t u = tid; u < n; u += st)
    if (rp[u + 1] < rp[u]) atomicOr(err, 1u);
  for (int64_t e = tid; e < m; e += st) {
    if (col[e] < 0 || col[e] >= n) atomicOr(err, 2u);
    if (w && w[e] == 0) atomicOr(err, 4u);
  }
  if (tid == 0 && (rp[0] != 0 || rp[n] != m)) atomicOr(err, 8u);
}

__global__ void k_max_u32(const uint32_t* __restrict__ w, int64_t m, unsigned int* __restrict__ out) {
  unsigned int mx = 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
    mx = max(mx, w[e]);
  mx = warp_max_u32(mx);
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(out, mx);
}

// (dst key, src value) per out-edge, plus the in-degree histogram; one warp
// per row keeps rows of any length coalesced
__global__ void k_csc_pairs(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj, int64_t n,
                            uint32_t* __restrict__ key, uint32_t* __restrict__ val, uint32_t* __restrict__ cnt) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int lane = threadIdx.x & 31;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    uint32_t a = rp[u], b = rp[u + 1];
    for (uint32_t e = a + lane; e < b; e += 32) {
      const uint32_t v = adj[e].x;
      key[e] = v;
      val[e] = (uint32_t)u;
      atomicAdd(&cnt[v], 1u);
    }
  }
}

// ------------------------------------------------------------------ host side

// GX_W_U8: 8-bit weights (a quarter of the PCIe bytes) widened on the device
__global__ void k_widen_u8(const uint8_t* __restrict__ in, uint32_t* __restrict__ out, int64_t m) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = in[i];
}

// the weights into g->in_w on stream st: a u32 copy, or (w8) a byte copy + widening
static void upload_weights(gx_graph* g, const uint32_t* w, bool w8, cudaMemcpyKind kind, cudaStream_t st) {
  Ctx* c = g->ctx;
  const int64_t m = g->m;
  if (!w8) {
    CUDA_OK(cudaMemcpyAsync(g->in_w.p, w, sizeof(uint32_t) * m, kind, st));
    return;
  }
  g->in_w8.alloc(c, (size_t)m);
  CUDA_OK(cudaMemcpyAsync(g->in_w8.p, w, (size_t)m, kind, st));
  k_widen_u8<<<grid_for(c, m), 256, 0, st>>>(g->in_w8.as<uint8_t>(), g->in_w.as<uint32_t>(), m);
  CUDA_OK(cudaGetLastError());
}

void device_upload_input(gx_graph* g, const int64_t* rp, const int32_t* col, const uint32_t* w,
                         bool device_ptrs, bool validate, bool async, bool w8) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  int64_t n = g->n, m = g->m;
  g->in_rp.alloc(c, sizeof(int64_t) * (n + 1));
  g->in_col.alloc(c, sizeof(int32_t) * std::max<int64_t>(m, 1));
  g->in_w.alloc(c, sizeof(uint32_t) * std::max<int64_t>(m, 1));
  cudaMemcpyKind kind = device_ptrs ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
  if (async && !device_ptrs && !validate && w && m > 0) {
    // row_ptr and col on the ctx stream; the weights (and their maximum) on
    // the copy stream once col has landed, so that work needing only the
    // structure (the blocked PageRank) overlaps their transfer
    if (!c->copy_stream) CUDA_OK(cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    g->maxw_buf.alloc(c, 16);
    CUDA_OK(cudaMemsetAsync(g->maxw_buf.p, 0, 16, s));
    CUDA_OK(cudaMemcpyAsync(g->in_rp.p, rp, sizeof(int64_t) * (n + 1), kind, s));
    CUDA_OK(cudaMemcpyAsync(g->in_col.p, col, sizeof(int32_t) * m, kind, s));
    cudaEvent_t ev;
    CUDA_OK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    CUDA_OK(cudaEventRecord(ev, s));
    CUDA_OK(cudaStreamWaitEvent(c->copy_stream, ev, 0));
    CUDA_OK(cudaEventDestroy(ev));
    upload_weights(g, w, w8, kind, c->copy_stream);
    k_max_u32<<<grid_for(c, m), 256, 0, c->copy_stream>>>(g->in_w.as<uint32_t>(), m, g->maxw_buf.as<unsigned int>());
    CUDA_OK(cudaGetLastError());
    g->maxw_pending = true;
    g->max_w = 1;   // until resolve_pending
    return;
  }
  CUDA_OK(cudaMemcpyAsync(g->in_rp.p, rp, sizeof(int64_t) * (n + 1), kind, s));
  if (m) {
    CUDA_OK(cudaMemcpyAsync(g->in_col.p, col, sizeof(int32_t) * m, kind, s));
    if (w) {
      upload_weights(g, w, w8, kind, s);
    } else {
      launch_fill_u32(c, g->in_w.as<uint32_t>(), 1u, m);  // all-ones weights
    }
  }
  DBuf scratch;
  scratch.alloc(c, 16);
  CUDA_OK(cudaMemsetAsync(scratch.p, 0, 16, s));
  unsigned int* err = scratch.as<unsigned int>();
  if (validate) {
    k_validate<<<grid_for(c, std::max(n, m)), 256, 0, s>>>(g->in_rp.as<int64_t>(), g->in_col.as<int32_t>(),
                                                           w ? g->in_w.as<uint32_t>() : nullptr, n, m, err);
  }
  if (m) k_max_u32<<<grid_for(c, m), 256, 0, s>>>(g->in_w.as<uint32_t>(), m, err + 1);
  CUDA_OK(cudaGetLastError());
  unsigned int h[2];
  CUDA_OK(cudaMemcpyAsync(h, err, 8, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  if (h[0] & 8u) GX_THROW(GX_E_INVALID, "row_ptr[0] must be 0 and row_ptr[n] == m");
  if (h[0] & 1u) GX_THROW(GX_E_INVALID, "row_ptr not monotone");
  if (h[0] & 2u) GX_THROW(GX_E_INVALID, "col out of range");
  if (h[0] & 4u) GX_THROW(GX_E_INVALID, "weight 0 (weights must be >= 1)");
  g->max_w = m ? std::max(1u, h[1]) : 1u;
}

static void build_csc_and_tiles(gx_graph* g) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  int64_t n = d.n_slots, m = d.m_slots;
  d.crp.alloc(c, sizeof(uint32_t) * (n + 1));
  d.csrc.alloc(c, sizeof(int32_t) * std::max<int64_t>(m, 1));
  if (m > 0) {
    // stable LSD radix sort of 32-bit dst keys carrying the src as payload:
    // edges enter in src order, so each CSC row comes out sorted by source
    DBuf k0, k1, v0, v1, tmp, cnt;
    k0.alloc(c, sizeof(uint32_t) * m);
    k1.alloc(c, sizeof(uint32_t) * m);
    v0.alloc(c, sizeof(uint32_t) * m);
    v1.alloc(c, sizeof(uint32_t) * m);
    cnt.alloc(c, sizeof(uint32_t) * (n + 1));
    CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * (n + 1), s));
    k_csc_pairs<<<grid_for(c, n * 32), 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), n, k0.as<uint32_t>(),
                                                    v0.as<uint32_t>(), cnt.as<uint32_t>());
    CUDA_OK(cudaGetLastError());
    int bits = 1;
    while ((int64_t(1) << bits) < n) bits++;
    size_t tb = 0;
    cub::DoubleBuffer<uint32_t> dk(k0.as<uint32_t>(), k1.as<uint32_t>()), dv(v0.as<uint32_t>(), v1.as<uint32_t>());
    CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, (int64_t)m, 0, bits, s));
    tmp.alloc(c, tb);
    CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, (int64_t)m, 0, bits, s));
    CUDA_OK(cudaMemcpyAsync(d.csrc.p, dv.Current(), sizeof(uint32_t) * m, cudaMemcpyDeviceToDevice, s));
    size_t sb = 0;
    CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, sb, cnt.as<uint32_t>(), d.crp.as<uint32_t>(), n + 1, s));
    DBuf t2;
    t2.alloc(c, sb);
    CUDA_OK(cub::DeviceScan::ExclusiveSum(t2.p, sb, cnt.as<uint32_t>(), d.crp.as<uint32_t>(), n + 1, s));
  } else {
    CUDA_OK(cudaMemsetAsync(d.crp.p, 0, sizeof(uint32_t) * (n + 1), s));
  }
  build_window_sell<uint32_t>(c, d.crp.as<uint32_t>(), reinterpret_cast<const uint32_t*>(d.csrc.p), n, PR_SENT,
                              d.pr_sell);
}

// ---- propagation-blocked PR layout (PbLayout, gx_internal.h) ----
// key = bin(v) * nb + block(u) per out-edge (sink-bin major), payload = the
// two local indices; histogram of keys for the segment offsets
__global__ void k_pb_pairs(const uint32_t* __restrict__ rp, const uint32_t* __restrict__ colp, uint32_t cstride,
                           int64_t n, uint32_t nb, uint32_t bblk,
                           uint32_t* __restrict__ key, uint32_t* __restrict__ val, uint32_t* __restrict__ cnt) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int lane = threadIdx.x & 31;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    const uint32_t a = rp[u], b = rp[u + 1];
    const uint32_t bu = (uint32_t)(u / PB_R), lu = (uint32_t)(u % PB_R);
    for (uint32_t e = a + lane; e < b; e += 32) {
      const uint32_t v = colp[(size_t)e * cstride];
      key[e] = ((v / PB_R) << bblk) | bu;
      val[e] = lu | ((v % PB_R) << 16);
      atomicAdd(&cnt[(v / PB_R) * nb + bu], 1u);
    }
  }
}
// the same with the edge's 8-bit weight in the payload's high word (weights
// resident and < 2^16): the sort then also yields the weights in blocked order
__global__ void k_pb_pairs_w(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj, int64_t n, uint32_t nb,
                             uint32_t bblk, uint32_t* __restrict__ key, unsigned long long* __restrict__ val,
                             uint32_t* __restrict__ cnt) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int lane = threadIdx.x & 31;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    const uint32_t a = rp[u], b = rp[u + 1];
    const uint32_t bu = (uint32_t)(u / PB_R), lu = (uint32_t)(u % PB_R);
    for (uint32_t e = a + lane; e < b; e += 32) {
      const uint2 vw = adj[e];
      key[e] = ((vw.x / PB_R) << bblk) | bu;
      val[e] = ((unsigned long long)vw.y << 32) | (lu | ((vw.x % PB_R) << 16));
      atomicAdd(&cnt[(vw.x / PB_R) * nb + bu], 1u);
    }
  }
}

// segment lengths padded to a multiple of PB_PAD (16-byte aligned u16 runs)
__global__ void k_pb_padcnt(const uint32_t* __restrict__ cnt, uint32_t* __restrict__ pc, int64_t nk) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nk; i += (int64_t)gridDim.x * blockDim.x)
    pc[i] = i + 1 < nk ? (cnt[i] + PB_PAD - 1) / PB_PAD * PB_PAD : 0u;
}

// element i of the sorted order (segment k = bin * nb + block) -> padded
// position P2[k] + (i - P[k])
template <class V>
__global__ void k_pb_place(const uint32_t* __restrict__ key, const V* __restrict__ pay,
                           const uint32_t* __restrict__ P, const uint32_t* __restrict__ P2, uint16_t* __restrict__ sl,
                           uint16_t* __restrict__ dl, uint16_t* __restrict__ w16, int64_t m, uint32_t nb,
                           uint32_t bblk) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t kk = key[i];
    const uint32_t k = (kk >> bblk) * nb + (kk & ((1u << bblk) - 1u));
    const V p = pay[i];
    const uint32_t pos = P2[k] + ((uint32_t)i - P[k]);
    sl[pos] = (uint16_t)(p & 0xffffu);
    dl[pos] = (uint16_t)((p >> 16) & 0xffffu);
    if constexpr (sizeof(V) == 8) {
      if (w16) w16[pos] = (uint16_t)(p >> 32);
    }
  }
}

// q[s*nb + b] = start of segment (s, b) = P2[b*nb + s]; row nb = bin ends
__global__ void k_pb_transpose(const uint32_t* __restrict__ P2, uint32_t* __restrict__ q, int64_t nb) {
  const int64_t tot = (nb + 1) * nb;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s = i / nb, b = i % nb;
    q[i] = s < nb ? P2[b * nb + s] : P2[(b + 1) * nb];
  }
}

void ensure_pb(gx_graph* g) {
  DevGraph& d = g->dg;
  PbLayout& L = d.pr_pb;
  if (L.built()) return;
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  const int64_t n = d.n_slots, m = d.m_slots;
  const int64_t nb = std::max<int64_t>(1, (n + PB_R - 1) / PB_R);
  const int64_t nk = nb * nb + 1;
  if (nb * nb >= (int64_t(1) << 32)) GX_THROW(GX_E_UNSUPPORTED, "graph too large for the blocked PR layout");
  L.nb = nb;
  DBuf P, P2, cnt, pc;
  cnt.alloc(c, sizeof(uint32_t) * nk);
  pc.alloc(c, sizeof(uint32_t) * nk);
  P.alloc(c, sizeof(uint32_t) * nk);
  P2.alloc(c, sizeof(uint32_t) * nk);
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * nk, s));
  // with resident 8-bit weights the sort carries them too (SSSP's dense
  // relaxation reads them in blocked order); an asynchronous upload's
  // blocked PageRank builds from col alone, and SSSP then runs without the
  // dense pass on this graph (it never gathers the weights at random)
  const bool with_w = d.max_w <= 0xffffu && !g->maxw_pending && m > 0;
  // key = bin << bblk | block; the edges arrive in CSR (= source block) order
  // and the radix sort is stable, so sorting the bin bits alone yields the
  // (bin, block) segment order: ceil(log2 nb) bits, 2 passes at RMAT-24/26
  // instead of 3 over the whole (bin, block) key
  int bits = 1;
  while ((int64_t(1) << bits) < nb) bits++;
  DBuf k0, k1, v0, v1, tmp;
  cub::DoubleBuffer<uint32_t> dk, dv;
  cub::DoubleBuffer<unsigned long long> dv64;
  if (m > 0) {
    k0.alloc(c, sizeof(uint32_t) * m);
    k1.alloc(c, sizeof(uint32_t) * m);
    v0.alloc(c, (with_w ? 8 : 4) * m);
    v1.alloc(c, (with_w ? 8 : 4) * m);

    size_t tb = 0;
    dk = cub::DoubleBuffer<uint32_t>(k0.as<uint32_t>(), k1.as<uint32_t>());
    if (with_w) {
      k_pb_pairs_w<<<grid_for(c, n * 32), 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), n, (uint32_t)nb,
                                                       (uint32_t)bits, k0.as<uint32_t>(), v0.as<unsigned long long>(),
                                                       cnt.as<uint32_t>());
      CUDA_OK(cudaGetLastError());
      dv64 = cub::DoubleBuffer<unsigned long long>(v0.as<unsigned long long>(), v1.as<unsigned long long>());
      CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv64, (int64_t)m, bits, 2 * bits, s));
      tmp.alloc(c, tb);
      CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv64, (int64_t)m, bits, 2 * bits, s));
    } else {
      // exact mode reads the uploaded col (not the {col, w} pairs, which an
      // asynchronous upload may still be producing)
      const bool ident = d.identity && g->in_col.p;
      k_pb_pairs<<<grid_for(c, n * 32), 256, 0, s>>>(d.rp.as<uint32_t>(),
                                                     ident ? g->in_col.as<uint32_t>() : d.adj.as<uint32_t>(),
                                                     ident ? 1u : 2u, n, (uint32_t)nb, (uint32_t)bits,
                                                     k0.as<uint32_t>(), v0.as<uint32_t>(), cnt.as<uint32_t>());
      CUDA_OK(cudaGetLastError());
      dv = cub::DoubleBuffer<uint32_t>(v0.as<uint32_t>(), v1.as<uint32_t>());
      CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, (int64_t)m, bits, 2 * bits, s));
      tmp.alloc(c, tb);
      CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, (int64_t)m, bits, 2 * bits, s));
    }
  }
  k_pb_padcnt<<<grid_for(c, nk), 256, 0, s>>>(cnt.as<uint32_t>(), pc.as<uint32_t>(), nk);
  size_t sb = 0;
  CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, sb, cnt.as<uint32_t>(), P.as<uint32_t>(), nk, s));
  DBuf t2;
  t2.alloc(c, sb);
  CUDA_OK(cub::DeviceScan::ExclusiveSum(t2.p, sb, cnt.as<uint32_t>(), P.as<uint32_t>(), nk, s));
  CUDA_OK(cub::DeviceScan::ExclusiveSum(t2.p, sb, pc.as<uint32_t>(), P2.as<uint32_t>(), nk, s));
  uint32_t mp = 0;
  CUDA_OK(cudaMemcpyAsync(&mp, P2.as<uint32_t>() + nb * nb, 4, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  if ((int64_t)mp < m || mp >= 0xfffffff0u) GX_THROW(GX_E_UNSUPPORTED, "padded edge count overflows 32 bits");
  L.m_pad = mp;
  const int64_t mm = std::max<int64_t>(mp, 8);
  L.src_loc.alloc(c, sizeof(uint16_t) * mm);
  L.dst_loc.alloc(c, sizeof(uint16_t) * mm);
  L.val.alloc(c, sizeof(float) * mm);
  if (with_w) {
    d.pb_w16.alloc(c, sizeof(uint16_t) * mm);
    CUDA_OK(cudaMemsetAsync(d.pb_w16.p, 0, sizeof(uint16_t) * mm, s));
  }
  // padding entries: source index PB_R (a zero term in shared memory), sink 0
  launch_fill_u32(c, L.src_loc.as<uint32_t>(), (uint32_t)PB_R * 0x10001u, mm / 2);   // mm is a multiple of 8
  CUDA_OK(cudaMemsetAsync(L.dst_loc.p, 0, sizeof(uint16_t) * mm, s));
  CUDA_OK(cudaMemsetAsync(L.val.p, 0, sizeof(float) * mm, s));
  if (m > 0)
  {
    if (with_w)
      k_pb_place<unsigned long long><<<grid_for(c, m), 256, 0, s>>>(dk.Current(), dv64.Current(), P.as<uint32_t>(),
                                                                    P2.as<uint32_t>(), L.src_loc.as<uint16_t>(),
                                                                    L.dst_loc.as<uint16_t>(), d.pb_w16.as<uint16_t>(), m,
                                                                    (uint32_t)nb, (uint32_t)bits);
    else
      k_pb_place<uint32_t><<<grid_for(c, m), 256, 0, s>>>(dk.Current(), dv.Current(), P.as<uint32_t>(),
                                                          P2.as<uint32_t>(), L.src_loc.as<uint16_t>(),
                                                          L.dst_loc.as<uint16_t>(), nullptr, m, (uint32_t)nb,
                                                          (uint32_t)bits);
  }
  L.q.alloc(c, sizeof(uint32_t) * (nb + 1) * nb);
  k_pb_transpose<<<grid_for(c, (nb + 1) * nb), 256, 0, s>>>(P2.as<uint32_t>(), L.q.as<uint32_t>(), nb);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));   // temporaries are freed on return
}

// ---- the edge weights in the blocked order (SSSP's dense relaxation, sssp.cu) ----
// true when the blocked layout carries them (built with resident weights < 2^16)
bool ensure_pb_w(gx_graph* g) {
  ensure_pb(g);
  return g->dg.pb_w16.p != nullptr;
}

// join the GX_ASYNC_UPLOAD work into the ctx stream; read the weights' maximum
void resolve_pending(gx_graph* g) {
  if (!g->ctx) return;
  cudaStream_t s = g->ctx->stream;
  if (g->pend_ev) {
    CUDA_OK(cudaStreamWaitEvent(s, g->pend_ev, 0));
    CUDA_OK(cudaEventDestroy(g->pend_ev));
    g->pend_ev = nullptr;
  }
  if (g->maxw_pending) {
    unsigned int h = 0;
    CUDA_OK(cudaMemcpyAsync(&h, g->maxw_buf.p, 4, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    g->max_w = std::max(1u, h);
    if (g->dg.identity) g->dg.max_w = g->max_w;
    g->maxw_pending = false;
  }
}

void ensure_csc(gx_graph* g) {
  if (g->dg.crp.p) return;
  build_csc_and_tiles(g);
}

void build_device_exact(gx_graph* g) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  DevGraph& d = g->dg;
  d = DevGraph();
  d.n = g->n;
  d.n_slots = g->n;
  d.m_slots = g->m;
  d.identity = true;
  d.max_w = g->max_w;
  int64_t n = d.n_slots, m = d.m_slots;
  d.rp.alloc(c, sizeof(uint32_t) * (n + 1));
  k_rp64_to_u32<<<grid_for(c, n + 1), 256, 0, s>>>(g->in_rp.as<int64_t>(), d.rp.as<uint32_t>(), n + 1);
  d.adj.alloc(c, sizeof(uint2) * std::max<int64_t>(m, 1));
  if (g->maxw_pending) {   // GX_ASYNC_UPLOAD: interleave behind the weights' copy
    cudaEvent_t ev;
    CUDA_OK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
    CUDA_OK(cudaEventRecord(ev, s));   // d.adj allocated
    CUDA_OK(cudaStreamWaitEvent(c->copy_stream, ev, 0));
    CUDA_OK(cudaEventDestroy(ev));
    k_interleave<<<grid_for(c, m), 256, 0, c->copy_stream>>>(g->in_col.as<int32_t>(), g->in_w.as<uint32_t>(),
                                                             d.adj.as<uint2>(), m);
    CUDA_OK(cudaGetLastError());
    CUDA_OK(cudaEventCreateWithFlags(&g->pend_ev, cudaEventDisableTiming));
    CUDA_OK(cudaEventRecord(g->pend_ev, c->copy_stream));
  } else if (m) {
    k_interleave<<<grid_for(c, m), 256, 0, s>>>(g->in_col.as<int32_t>(), g->in_w.as<uint32_t>(), d.adj.as<uint2>(),
                                                m);
  }
  d.D.alloc(c, sizeof(uint32_t) * std::max<int64_t>(n, 1));
  k_outdeg<<<grid_for(c, n), 256, 0, s>>>(d.rp.as<uint32_t>(), d.D.as<uint32_t>(), n);
  CUDA_OK(cudaGetLastError());
}

// Upload the host slot graph produced by transform_host.
void build_device_slots(gx_graph* g) {
  Ctx* c = g->ctx;
  cudaStream_t s = c->stream;
  const SlotGraph& sg = g->sg;
  DevGraph& d = g->dg;
  d = DevGraph();
  d.n = sg.n;
  d.n_slots = sg.n_slots;
  d.m_slots = sg.m_slots;
  d.identity = false;
  int64_t n = sg.n_slots, m = sg.m_slots;
  if (m >= (int64_t(1) << 32) - 1) GX_THROW(GX_E_UNSUPPORTED, "m' must be < 2^32 - 1");
  std::vector<uint32_t> rp32(n + 1);
  for (int64_t i = 0; i <= n; i++) rp32[i] = (uint32_t)sg.rp[i];
  std::vector<uint2> adj(std::max<int64_t>(m, 1));
  uint32_t mw = 1;
  for (int64_t e = 0; e < m; e++) {
    adj[e] = make_uint2((uint32_t)sg.col[e], sg.w[e]);
    mw = std::max(mw, sg.w[e]);
  }
  d.max_w = mw;
  // logical out-degree per vertex, summed over its copies
  std::vector<uint32_t> ldeg(sg.n, 0), D(std::max<int64_t>(n, 1), 0);
  for (int64_t sl = 0; sl < n; sl++)
    if (sg.kind[sl] != HOLE) ldeg[sg.slot_to_orig[sl]] += (uint32_t)(sg.rp[sl + 1] - sg.rp[sl]);
  for (int64_t sl = 0; sl < n; sl++)
    if (sg.kind[sl] != HOLE) D[sl] = ldeg[sg.slot_to_orig[sl]];
  // groups: owner first, then replica slots ascending
  std::vector<std::vector<int32_t>> rep(sg.n);
  for (int64_t sl = 0; sl < n; sl++)
    if (sg.kind[sl] == REPLICA) rep[sg.slot_to_orig[sl]].push_back((int32_t)sl);
  std::vector<int32_t> gptr{0}, gslots, gid(std::max<int64_t>(n, 1), -1);
  std::vector<int32_t> gown;
  for (int64_t v = 0; v < sg.n; v++) {
    if (rep[v].empty()) continue;
    int32_t gi = (int32_t)gown.size();
    gown.push_back(sg.owner_slot[v]);
    gslots.push_back(sg.owner_slot[v]);
    gid[sg.owner_slot[v]] = gi;
    for (int32_t r : rep[v]) {
      gslots.push_back(r);
      gid[r] = gi;
    }
    gptr.push_back((int32_t)gslots.size());
  }
  d.n_groups = (int64_t)gown.size();
  d.n_gslots = (int64_t)gslots.size();
  // in-edges of each group's owner slot: (src slot, w)
  std::vector<int32_t> gin_ptr(d.n_groups + 1, 0);
  std::vector<uint2> gin;
  if (d.n_groups) {
    std::vector<std::vector<uint2>> tmp(d.n_groups);
    for (int64_t sl = 0; sl < n; sl++)
      for (int64_t e = sg.rp[sl]; e < sg.rp[sl + 1]; e++) {
        int32_t q = sg.col[e];
        if (gid[q] >= 0 && gown[gid[q]] == q) tmp[gid[q]].push_back(make_uint2((uint32_t)sl, sg.w[e]));
      }
    for (int64_t gi = 0; gi < d.n_groups; gi++) {
      gin_ptr[gi + 1] = gin_ptr[gi] + (int32_t)tmp[gi].size();
      gin.insert(gin.end(), tmp[gi].begin(), tmp[gi].end());
    }
  }
  auto up = [&](DBuf& b, const void* src, size_t bytes) {
    b.alloc(c, std::max<size_t>(bytes, 16));
    if (bytes) CUDA_OK(cudaMemcpyAsync(b.p, src, bytes, cudaMemcpyHostToDevice, s));
  };
  up(d.rp, rp32.data(), sizeof(uint32_t) * (n + 1));
  up(d.adj, adj.data(), sizeof(uint2) * m);
  up(d.D, D.data(), sizeof(uint32_t) * n);
  up(d.owner, sg.owner_slot.data(), sizeof(int32_t) * sg.n);
  up(d.kind, sg.kind.data(), n);
  if (d.n_groups) {
    up(d.gid, gid.data(), sizeof(int32_t) * n);
    up(d.gptr, gptr.data(), sizeof(int32_t) * gptr.size());
    up(d.gslots, gslots.data(), sizeof(int32_t) * gslots.size());
    up(d.g_in_ptr, gin_ptr.data(), sizeof(int32_t) * gin_ptr.size());
    up(d.g_in, gin.data(), sizeof(uint2) * gin.size());
  }
  // §3 tiles: members as owner slots + local CSR (u8 member indices)
  int64_t nt = (int64_t)sg.tile_centre.size();
  d.n_tiles = nt;
  if (nt) {
    std::vector<int32_t> tp(nt + 1, 0), tmem, teptr(nt + 1, 0), titers(nt);
    std::vector<uint2> tedges;  // {src_local | dst_local << 8, w}
    for (int64_t t = 0; t < nt; t++) {
      std::vector<int32_t> mem;
      for (int64_t i = sg.tile_ptr[t]; i < sg.tile_ptr[t + 1]; i++) mem.push_back(sg.owner_slot[sg.tile_members[i]]);
      std::sort(mem.begin(), mem.end());
      for (size_t a = 0; a < mem.size(); a++) {
        int32_t sl = mem[a];
        for (int64_t e = sg.rp[sl]; e < sg.rp[sl + 1]; e++) {
          auto it = std::lower_bound(mem.begin(), mem.end(), sg.col[e]);
          if (it != mem.end() && *it == sg.col[e]) {
            uint32_t b = (uint32_t)(it - mem.begin());
            tedges.push_back(make_uint2((uint32_t)a | (b << 8), sg.w[e]));
          }
        }
      }
      tmem.insert(tmem.end(), mem.begin(), mem.end());
      tp[t + 1] = (int32_t)tmem.size();
      teptr[t + 1] = (int32_t)tedges.size();
      titers[t] = sg.tile_iters[t];
      d.t_max_members = std::max<int64_t>(d.t_max_members, (int64_t)mem.size());
      d.t_max_edges = std::max<int64_t>(d.t_max_edges, teptr[t + 1] - teptr[t]);
    }
    up(d.t_ptr, tp.data(), sizeof(int32_t) * tp.size());
    up(d.t_members, tmem.data(), sizeof(int32_t) * tmem.size());
    up(d.t_eptr, teptr.data(), sizeof(int32_t) * teptr.size());
    up(d.t_edges, tedges.data(), sizeof(uint2) * tedges.size());
    up(d.t_iters, titers.data(), sizeof(int32_t) * titers.size());
    // slot -> tile map and the touched-tile scratch of the SSSP local pass
    std::vector<int32_t> st(sg.n_slots, -1);
    for (int64_t t = 0; t < nt; t++)
      for (int32_t i = tp[t]; i < tp[t + 1]; i++) st[tmem[i]] = (int32_t)t;
    up(d.slot_tile, st.data(), sizeof(int32_t) * st.size());
    std::vector<uint32_t> zero((nt + 31) / 32, 0u);
    up(d.tile_mark, zero.data(), sizeof(uint32_t) * zero.size());
    d.tile_list.alloc(c, sizeof(int32_t) * nt);
  }
  if (!sg.sched.empty()) up(d.sched, sg.sched.data(), sizeof(int32_t) * sg.sched.size());
  CUDA_OK(cudaStreamSynchronize(s));  // host vectors go out of scope
}

}  // namespace gx

// ---- rank-local PageRank layout of the partitioned path (dist.h) ----
namespace gx {

__global__ void k_indeg(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj, int64_t n,
                        uint32_t* __restrict__ cnt) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw)
    for (uint32_t e = rp[u] + lane_id(); e < rp[u + 1]; e += 32) atomicAdd(&cnt[adj[e].x], 1u);
}
// (dst << 32 | src) per out-edge, in source order
__global__ void k_pairs_u64(const uint32_t* __restrict__ rp, const uint2* __restrict__ adj, int64_t n,
                            unsigned long long* __restrict__ out) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw)
    for (uint32_t e = rp[u] + lane_id(); e < rp[u + 1]; e += 32)
      out[e] = ((unsigned long long)adj[e].x << 32) | (unsigned long long)u;
}
__global__ void k_rebase_u32(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, int64_t n1) {
  const uint32_t b = in[0];
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n1; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = in[i] - b;
}
__global__ void k_lo32(const unsigned long long* __restrict__ in, uint32_t* __restrict__ out, int64_t m) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (uint32_t)in[i];
}
struct DstInRange {
  unsigned long long lo, hi;
  __host__ __device__ bool operator()(const unsigned long long& p) const {
    const unsigned long long d = p >> 32;
    return d >= lo && d < hi;
  }
};

// In-CSC of rows [lo, hi) for each rank (all P when `all`, else this rank),
// balanced by in-edges: the (dst, src) pairs with dst in the range are
// selected in source order and stably sorted by dst, so each local row lists
// its sources ascending (the same order as the full CSC); the windowed SELL-32
// is built over the local rows.  Only the slices stay resident.
RankLayouts& ensure_pr_ranks(gx_graph* g, int P, bool all) {
  DevGraph& d = g->dg;
  RankLayouts& L = d.rk_pr;
  Ctx* c = g->ctx;
  const int want_rank = all ? -1 : c->rank;
  if (L.P == P && L.rank == want_rank) return L;
  L = RankLayouts();
  cudaStream_t s = c->stream;
  const int64_t n = d.n_slots, m = d.m_slots;
  DBuf cnt, crp;
  cnt.alloc(c, sizeof(uint32_t) * (n + 1));
  crp.alloc(c, sizeof(uint32_t) * (n + 1));
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint32_t) * (n + 1), s));
  if (m) k_indeg<<<grid_for(c, n * 32), 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), n, cnt.as<uint32_t>());
  {
    size_t tb = 0;
    CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt.as<uint32_t>(), crp.as<uint32_t>(), n + 1, s));
    DBuf t;
    t.alloc(c, tb);
    CUDA_OK(cub::DeviceScan::ExclusiveSum(t.p, tb, cnt.as<uint32_t>(), crp.as<uint32_t>(), n + 1, s));
  }
  cnt.reset();
  std::vector<uint32_t> hcrp(n + 1);
  CUDA_OK(cudaMemcpyAsync(hcrp.data(), crp.p, sizeof(uint32_t) * (n + 1), cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  L.bounds = partition_rows(std::vector<int64_t>(hcrp.begin(), hcrp.end()), n, P, PRW_ALIGN);
  L.P = P;
  L.rank = want_rank;
  DBuf pairs;
  pairs.alloc(c, sizeof(unsigned long long) * std::max<int64_t>(m, 1));
  if (m) k_pairs_u64<<<grid_for(c, n * 32), 256, 0, s>>>(d.rp.as<uint32_t>(), d.adj.as<uint2>(), n,
                                                         pairs.as<unsigned long long>());
  int bits = 1;
  while ((int64_t(1) << bits) < n) bits++;
  for (int p = 0; p < P; p++) {
    if (!all && p != c->rank) continue;
    RankSlice sl;
    sl.lo = L.bounds[p];
    sl.hi = L.bounds[p + 1];
    const int64_t nl = sl.hi - sl.lo;
    sl.m = (int64_t)hcrp[sl.hi] - (int64_t)hcrp[sl.lo];
    sl.crp.alloc(c, sizeof(uint32_t) * (nl + 1));
    k_rebase_u32<<<grid_for(c, nl + 1), 256, 0, s>>>(crp.as<uint32_t>() + sl.lo, sl.crp.as<uint32_t>(), nl + 1);
    sl.csrc.alloc(c, sizeof(int32_t) * std::max<int64_t>(sl.m, 1));
    if (sl.m) {
      DBuf sel, sel2, nsel, tmp;
      sel.alloc(c, sizeof(unsigned long long) * sl.m);
      sel2.alloc(c, sizeof(unsigned long long) * sl.m);
      nsel.alloc(c, 8);
      size_t tb = 0;
      DstInRange pred{(unsigned long long)sl.lo, (unsigned long long)sl.hi};
      CUDA_OK(cub::DeviceSelect::If(nullptr, tb, pairs.as<unsigned long long>(), sel.as<unsigned long long>(),
                                    nsel.as<int64_t>(), m, pred, s));
      tmp.alloc(c, tb);
      CUDA_OK(cub::DeviceSelect::If(tmp.p, tb, pairs.as<unsigned long long>(), sel.as<unsigned long long>(),
                                    nsel.as<int64_t>(), m, pred, s));
      cub::DoubleBuffer<unsigned long long> kb(sel.as<unsigned long long>(), sel2.as<unsigned long long>());
      size_t sb = 0;
      CUDA_OK(cub::DeviceRadixSort::SortKeys(nullptr, sb, kb, sl.m, 32, 32 + bits, s));
      DBuf t2;
      t2.alloc(c, sb);
      CUDA_OK(cub::DeviceRadixSort::SortKeys(t2.p, sb, kb, sl.m, 32, 32 + bits, s));
      k_lo32<<<grid_for(c, sl.m), 256, 0, s>>>(kb.Current(), reinterpret_cast<uint32_t*>(sl.csrc.p), sl.m);
      CUDA_OK(cudaGetLastError());
      CUDA_OK(cudaStreamSynchronize(s));   // the scratch buffers go out of scope
    }
    build_window_sell<uint32_t>(c, sl.crp.as<uint32_t>(), reinterpret_cast<const uint32_t*>(sl.csrc.p), nl, PR_SENT,
                                sl.sell);
    L.r.push_back(std::move(sl));
  }
  CUDA_OK(cudaStreamSynchronize(s));
  return L;
}

}  // namespace gx
