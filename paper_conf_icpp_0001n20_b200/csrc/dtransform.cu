// dtransform.cu -- the device-resident slot graph of the Graffix transforms
// ("relabel and CSR rebuild, all on device. Keep host
// code only for the sequential cursor numbering and greedy budgeted
// insertion"; PAPER.md P@41797, P@46748-46927: the preprocessing cost that the
// amortisation argument rests on).
//
// The slot graph under construction is one flat edge list in HBM,
//   key = src slot << 32 | dst slot,   val = weight | AddKind << 32,
// and every bulk step of transform.cpp's host pipeline becomes a pass over it:
//   §2 relabel (Alg 2 l.10-20 applied to the edges), replica candidates
//      (Alg 2 l.21-27: count_n[C] per (slot, chunk) run of a sorted row),
//      replica rows (l.28-35: moved edges re-homed, 2-hop edges into C with
//      the minimum path weight, R16/R17);
//   §3 the logical graph G_L (original ids) and its undirected view U, the
//      input of the clustering coefficient (P@29857) and the greedy insertion;
//   §4 degree buckets and the warp schedule (P@33145-33432: a stable radix
//      sort on the bucket), the padded vertices of each warp (P@33654-35029),
//      their 2-hop candidates (gtransform.cu);
//   assembly: one radix sort by (src, dst) gives the slot CSR with rows sorted
//      by destination (R11).
// The sequential decisions (cursor numbering, the choice of the h best
// replica candidates of a level, the §3 budgeted insertion and subgraph
// packing) stay host C++ in transform.cpp, which drives these passes
// (transform_device).  Results equal the host pipeline's bit for bit
// (tests/test_gpu_transform.py compares both with the oracle and each other).
#include <cub/cub.cuh>

#include <algorithm>
#include <cstring>
#include <vector>

#include "gx_internal.h"
#include "kernels_common.cuh"

namespace gx {

namespace {

__device__ __forceinline__ uint32_t ksrc(unsigned long long k) { return (uint32_t)(k >> 32); }
__device__ __forceinline__ uint32_t kdst(unsigned long long k) { return (uint32_t)k; }

__device__ __forceinline__ uint32_t combine_w_d(uint32_t w1, uint32_t w2, int rule) {
  if (rule == GX_W_MAX) return max(w1, w2);
  if (rule == GX_W_MEAN) return max(1u, (uint32_t)(((uint64_t)w1 + w2) / 2));
  return w1 + w2;   // P@34493, R17: the 2-hop path's total weight
}

// first e in [lo, hi) with key[e] >= x (rows sorted by key)
__device__ __forceinline__ int64_t lower_bound_u64(const unsigned long long* __restrict__ key, int64_t lo, int64_t hi,
                                                   unsigned long long x) {
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (key[mid] < x) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

int slot_bits(int64_t ns) {
  int b = 1;
  while (b < 32 && ((int64_t)1 << b) < ns) b++;
  return b;
}

// ---- edge list from the canonical CSR, relabelled by nw (identity if null)
__global__ void k_dt_from_csr(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                              const uint32_t* __restrict__ w, const int32_t* __restrict__ nw, int64_t n,
                              unsigned long long* __restrict__ key, unsigned long long* __restrict__ val) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nwp = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nwp) {
    const unsigned long long su = (unsigned long long)(uint32_t)(nw ? nw[u] : (int32_t)u) << 32;
    for (int64_t e = rp[u] + lane; e < rp[u + 1]; e += 32) {
      const int32_t v = col[e];
      key[e] = su | (uint32_t)(nw ? nw[v] : v);
      val[e] = w[e];   // AddKind ADD_NONE
    }
  }
}

// rp[x] = first edge of row x in a key-sorted list (rows with no edge get the
// next row's start); O(ns + m) over all threads
__global__ void k_dt_rowptr(const unsigned long long* __restrict__ key, int64_t m, int64_t ns,
                            int64_t* __restrict__ rp) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e <= m; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = e == 0 ? 0 : (int64_t)ksrc(key[e - 1]) + 1;
    const int64_t hi = e == m ? ns : (int64_t)ksrc(key[e]);
    for (int64_t x = lo; x <= hi; x++) rp[x] = e;
  }
}

// ---- §2 replica candidates: one thread per (slot, chunk) run of the sorted rows
__global__ void k_dt_rep_cand(const unsigned long long* __restrict__ key, int64_t m, int k,
                              const int32_t* __restrict__ chunk_lv, const int32_t* __restrict__ nonhole,
                              int64_t theta_ppm, int4* __restrict__ out, unsigned long long* __restrict__ cnt) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long ke = key[e];
    const uint32_t s = ksrc(ke), C = kdst(ke) / (uint32_t)k;
    const int32_t lv = chunk_lv[C];
    if (lv < 0) continue;
    if (e > 0 && ksrc(key[e - 1]) == s && kdst(key[e - 1]) / (uint32_t)k == C) continue;
    int64_t c = 1;
    while (e + c < m && ksrc(key[e + c]) == s && kdst(key[e + c]) / (uint32_t)k == C) c++;
    // Alg 2 l.24: count_n[C] / nonhole(C) >= theta_conn, compared in ppm
    if (c * 1000000 < theta_ppm * (int64_t)nonhole[C]) continue;
    const unsigned long long i = atomicAdd(cnt, 1ull);
    if (out) out[i] = make_int4(lv, (int)c, (int)s, (int)C);
  }
}

// ---- §2 replica rows (Alg 2 l.28-35, R16/R17): warp per assignment (s, C,
// hole).  The 2-hop paths s -> x -> q (q in chunk C) use the pre-move rows;
// each q keeps its lightest combined weight (shared atomicMin over the k <= 32
// slots of C); q must not be s, a hole, or already an out-neighbour of s.
__global__ void k_dt_replicate(const unsigned long long* __restrict__ key, const unsigned long long* __restrict__ val,
                               const int64_t* __restrict__ rp, const int4* __restrict__ asg, int64_t na, int k,
                               const uint8_t* __restrict__ kind, int rule, unsigned long long* __restrict__ okey,
                               unsigned long long* __restrict__ oval, unsigned long long* __restrict__ ocnt,
                               longlong2* __restrict__ mrange) {
  __shared__ uint32_t best[8][32];
  __shared__ uint32_t seen[8];   // q reached by some path (a path weight may equal INF)
  const unsigned lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwp = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t ai = warp; ai < na; ai += nwp) {
    const int4 a = asg[ai];   // (s, C, hole lo, hole hi)
    const uint32_t s = (uint32_t)a.x, C = (uint32_t)a.y;
    const uint64_t hole = (uint64_t)(uint32_t)a.z | ((uint64_t)(uint32_t)a.w << 32);
    const uint32_t c0 = C * (uint32_t)k, c1 = c0 + (uint32_t)k;
    best[wib][lane] = INF;
    if (lane == 0) {
      seen[wib] = 0;
      // s's edges into C, found before any row is re-homed (k_dt_move: two
      // assignments of one slot must not search a row the other is editing)
      const unsigned long long kb = (unsigned long long)s << 32;
      mrange[ai] = make_longlong2(lower_bound_u64(key, rp[s], rp[s + 1], kb | c0),
                                  lower_bound_u64(key, rp[s], rp[s + 1], kb | c1));
    }
    __syncwarp();
    uint32_t mask = 0;
    for (int64_t ev = rp[s] + lane; ev < rp[s + 1]; ev += 32) {
      const uint32_t x = kdst(key[ev]);
      const uint32_t w1 = (uint32_t)val[ev];
      if (x >= c0 && x < c1) mask |= 1u << (x - c0);
      const int64_t xe = rp[x + 1];
      for (int64_t j = lower_bound_u64(key, rp[x], xe, ((unsigned long long)x << 32) | c0); j < xe; j++) {
        const uint32_t q = kdst(key[j]);
        if (q >= c1) break;
        atomicMin(&best[wib][q - c0], combine_w_d(w1, (uint32_t)val[j], rule));
        atomicOr(&seen[wib], 1u << (q - c0));
      }
    }
    mask = __reduce_or_sync(FULL, mask);
    __syncwarp();
    const uint32_t q = c0 + lane;
    const uint32_t b = best[wib][lane];
    const bool emit = lane < (unsigned)k && ((seen[wib] >> lane) & 1u) && !((mask >> lane) & 1u) && q != s && kind[q] != HOLE;
    const unsigned bal = __ballot_sync(FULL, emit);
    unsigned long long base = 0;
    if (lane == 0 && bal) base = atomicAdd(ocnt, (unsigned long long)__popc(bal));
    base = __shfl_sync(FULL, base, 0);
    if (emit) {
      const unsigned long long o = base + __popc(bal & lanemask_lt());
      okey[o] = (hole << 32) | q;
      oval[o] = (unsigned long long)b | ((unsigned long long)ADD_COALESCE << 32);
    }
    __syncwarp();
  }
}

// the moved edges (s's edges into C, ranges recorded by k_dt_replicate)
// re-homed on the replica slot
__global__ void k_dt_move(unsigned long long* __restrict__ key, const longlong2* __restrict__ mrange,
                          const int4* __restrict__ asg, int64_t na) {
  const unsigned lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwp = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t ai = warp; ai < na; ai += nwp) {
    const int4 a = asg[ai];
    const unsigned long long hole = (unsigned long long)(uint32_t)a.z | ((unsigned long long)(uint32_t)a.w << 32);
    const longlong2 r = mrange[ai];
    for (int64_t e = r.x + lane; e < r.y; e += 32) key[e] = (hole << 32) | kdst(key[e]);
  }
}

// ---- §3 / §4 logical graph G_L: every slot edge in original ids
__global__ void k_dt_logical(const unsigned long long* __restrict__ key, const unsigned long long* __restrict__ val,
                             int64_t m, const int32_t* __restrict__ s2o, unsigned long long* __restrict__ lkey,
                             unsigned long long* __restrict__ lval) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = key[e];
    lkey[e] = ((unsigned long long)(uint32_t)s2o[ksrc(k)] << 32) | (uint32_t)s2o[kdst(k)];
    lval[e] = (uint32_t)val[e];
  }
}

__global__ void k_dt_split(const unsigned long long* __restrict__ key, const unsigned long long* __restrict__ val,
                           int64_t m, int32_t* __restrict__ dst, uint32_t* __restrict__ w, uint8_t* __restrict__ add) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long v = val[e];
    if (dst) dst[e] = (int32_t)kdst(key[e]);
    if (w) w[e] = (uint32_t)v;
    if (add) add[e] = (uint8_t)(v >> 32);
  }
}

__global__ void k_dt_pairs(const int32_t* __restrict__ d, const uint32_t* __restrict__ w, int64_t m,
                           unsigned long long* __restrict__ out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
    out[e] = ((unsigned long long)w[e] << 32) | (uint32_t)d[e];
}

// U: both directions of every G_L edge (sorted + deduplicated by the caller)
__global__ void k_dt_sym(const unsigned long long* __restrict__ lkey, int64_t m, unsigned long long* __restrict__ ukey) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = lkey[e];
    ukey[2 * e] = k;
    ukey[2 * e + 1] = ((unsigned long long)kdst(k) << 32) | ksrc(k);
  }
}

// ---- §4: degree buckets (R30: 0 for d = 0, else 1 + floor(log2 d)), descending
__global__ void k_dt_bucket_key(const int64_t* __restrict__ rp, const int32_t* __restrict__ sl, int64_t no,
                                uint32_t* __restrict__ bkey) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < no; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t s = sl[i];
    const uint64_t d = (uint64_t)(rp[s + 1] - rp[s]);
    const uint32_t b = d ? 64u - (uint32_t)__clzll((long long)d) : 0u;
    bkey[i] = 255u - b;
  }
}

__global__ void k_dt_nonhole_flag(const uint8_t* __restrict__ kind, int64_t ns, int32_t* __restrict__ idx,
                                  uint8_t* __restrict__ flag) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < ns; s += (int64_t)gridDim.x * blockDim.x) {
    idx[s] = (int32_t)s;
    flag[s] = kind[s] != HOLE;
  }
}

// P@33654-35029 (R31-R33): in each warp of the schedule, M = max out-degree;
// an owner slot with 0 < d < M, 1 - d/M < theta_d and d < ceil(f M) is padded
// towards ceil(f M).  One thread per schedule entry; the warp of the schedule
// is the hardware warp (entries 32-aligned).  Queries appended (order free:
// the added edges are sorted into their rows by the assembly).
__global__ void k_dt_pad_query(const int64_t* __restrict__ rp, const int32_t* __restrict__ order, int64_t no,
                               const uint8_t* __restrict__ kind, const int32_t* __restrict__ s2o, int64_t th,
                               int64_t f, int32_t* __restrict__ qs, int32_t* __restrict__ qu,
                               int32_t* __restrict__ qtake, unsigned long long* __restrict__ qcnt) {
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  const int64_t span = (no + 31) / 32 * 32;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < span; i += nthr) {
    int32_t s = -1;
    uint32_t d = 0;
    if (i < no) {
      s = order[i];
      d = (uint32_t)(rp[s + 1] - rp[s]);
    }
    const int64_t M = (int64_t)__reduce_max_sync(FULL, d);
    const int64_t target = (f * M + 999999) / 1000000;
    const int64_t dd = d;
    const bool q = s >= 0 && kind[s] == OWNER && 0 < dd && dd < M && (M - dd) * 1000000 < th * M && dd < target;
    const unsigned bal = __ballot_sync(FULL, q);
    unsigned long long base = 0;
    if ((threadIdx.x & 31) == 0 && bal) base = atomicAdd(qcnt, (unsigned long long)__popc(bal));
    base = __shfl_sync(FULL, base, 0);
    if (q) {
      const unsigned long long o = base + __popc(bal & lanemask_lt());
      qs[o] = s;
      qu[o] = s2o[s];
      qtake[o] = (int32_t)(target - dd);
    }
  }
}

template <class T>
void upload(Ctx* c, DBuf& b, const T* h, int64_t n) {
  b.alloc(c, sizeof(T) * std::max<int64_t>(n, 1));
  if (n) CUDA_OK(cudaMemcpyAsync(b.p, h, sizeof(T) * n, cudaMemcpyHostToDevice, c->stream));
}

// radix sort of (key, val) pairs over the low `bits` of the key, in place
void sort_pairs(Ctx* c, DBuf& key, DBuf& val, int64_t m, int bits) {
  if (m <= 1) return;
  cudaStream_t s = c->stream;
  DBuf k1, v1, tmp;
  k1.alloc(c, sizeof(uint64_t) * m);
  v1.alloc(c, sizeof(uint64_t) * m);
  cub::DoubleBuffer<uint64_t> dk(key.as<uint64_t>(), k1.as<uint64_t>());
  cub::DoubleBuffer<uint64_t> dv(val.as<uint64_t>(), v1.as<uint64_t>());
  size_t tb = 0;
  CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, m, 0, bits, s));
  tmp.alloc(c, tb);
  CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, m, 0, bits, s));
  if (dk.Current() != key.as<uint64_t>()) std::swap(key, k1);
  if (dv.Current() != val.as<uint64_t>()) std::swap(val, v1);
}

int64_t read_count(Ctx* c, const DBuf& cnt) {
  unsigned long long h = 0;
  CUDA_OK(cudaMemcpyAsync(&h, cnt.p, 8, cudaMemcpyDeviceToHost, c->stream));
  CUDA_OK(cudaStreamSynchronize(c->stream));
  return (int64_t)h;
}

}  // namespace

void dt_from_csr(Ctx* c, const HostCSR& g, const int32_t* nw, DEdges& E, const int64_t* drp, const int32_t* dcol,
                 const uint32_t* dw) {
  cudaStream_t s = c->stream;
  DBuf rp, col, w, dnw;
  if (!drp) {   // no resident copy: upload the canonical graph
    upload(c, rp, g.rp.data(), g.n + 1);
    upload(c, col, g.col.data(), g.m);
    upload(c, w, g.w.data(), g.m);
    drp = rp.as<int64_t>();
    dcol = col.as<int32_t>();
    dw = w.as<uint32_t>();
  }
  if (nw) upload(c, dnw, nw, g.n);
  E.m = g.m;
  E.key.alloc(c, sizeof(uint64_t) * std::max<int64_t>(g.m, 1));
  E.val.alloc(c, sizeof(uint64_t) * std::max<int64_t>(g.m, 1));
  k_dt_from_csr<<<c->num_sms * 16, 256, 0, s>>>(drp, dcol, dw, nw ? dnw.as<int32_t>() : nullptr, g.n,
                                                 E.key.as<unsigned long long>(), E.val.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));   // the host staging buffers go out of scope
}

void dt_sort(Ctx* c, DEdges& E, int64_t ns) { sort_pairs(c, E.key, E.val, E.m, 32 + slot_bits(ns)); }

void dt_row_ptr(Ctx* c, const DEdges& E, int64_t ns, DBuf& rp) {
  rp.alloc(c, sizeof(int64_t) * (ns + 1));
  k_dt_rowptr<<<grid_for(c, E.m + 1), 256, 0, c->stream>>>(E.key.as<unsigned long long>(), E.m, ns, rp.as<int64_t>());
  CUDA_OK(cudaGetLastError());
}

void dt_replica_candidates(Ctx* c, const DEdges& E, int k, const std::vector<int32_t>& chunk_lv,
                           const std::vector<int32_t>& nonhole, int64_t theta_ppm, std::vector<DtCand>& out) {
  out.clear();
  if (E.m == 0) return;
  cudaStream_t s = c->stream;
  DBuf dlv, dnh, cnt, buf;
  upload(c, dlv, chunk_lv.data(), (int64_t)chunk_lv.size());
  upload(c, dnh, nonhole.data(), (int64_t)nonhole.size());
  cnt.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, 8, s));
  const int grid = grid_for(c, E.m);
  k_dt_rep_cand<<<grid, 256, 0, s>>>(E.key.as<unsigned long long>(), E.m, k, dlv.as<int32_t>(), dnh.as<int32_t>(),
                                     theta_ppm, nullptr, cnt.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  const int64_t nc = read_count(c, cnt);
  if (nc == 0) return;
  buf.alloc(c, sizeof(int4) * nc);
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, 8, s));
  k_dt_rep_cand<<<grid, 256, 0, s>>>(E.key.as<unsigned long long>(), E.m, k, dlv.as<int32_t>(), dnh.as<int32_t>(),
                                     theta_ppm, buf.as<int4>(), cnt.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  out.resize(nc);
  static_assert(sizeof(DtCand) == sizeof(int4), "DtCand is (lv, cnt, s, C)");
  CUDA_OK(cudaMemcpyAsync(out.data(), buf.p, sizeof(int4) * nc, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
}

int64_t dt_replicate(Ctx* c, DEdges& E, int64_t ns, int k, const std::vector<DtAsg>& asg,
                     const std::vector<uint8_t>& kind, int rule) {
  const int64_t na = (int64_t)asg.size();
  if (na == 0) return 0;
  cudaStream_t s = c->stream;
  DBuf rp, dasg, dkind, okey, oval, cnt, mr;
  dt_row_ptr(c, E, ns, rp);
  mr.alloc(c, sizeof(longlong2) * na);
  std::vector<int4> ha(na);
  for (int64_t i = 0; i < na; i++)
    ha[i] = make_int4(asg[i].s, asg[i].C, (int)(uint32_t)asg[i].hole, (int)(uint32_t)((uint64_t)asg[i].hole >> 32));
  upload(c, dasg, ha.data(), na);
  upload(c, dkind, kind.data(), (int64_t)kind.size());
  okey.alloc(c, sizeof(uint64_t) * na * k);
  oval.alloc(c, sizeof(uint64_t) * na * k);
  cnt.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, 8, s));
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((na + 7) / 8, c->num_sms * 16));
  k_dt_replicate<<<grid, 256, 0, s>>>(E.key.as<unsigned long long>(), E.val.as<unsigned long long>(),
                                      rp.as<int64_t>(), dasg.as<int4>(), na, k, dkind.as<uint8_t>(), rule,
                                      okey.as<unsigned long long>(), oval.as<unsigned long long>(),
                                      cnt.as<unsigned long long>(), mr.as<longlong2>());
  CUDA_OK(cudaGetLastError());
  k_dt_move<<<grid, 256, 0, s>>>(E.key.as<unsigned long long>(), mr.as<longlong2>(), dasg.as<int4>(), na);
  CUDA_OK(cudaGetLastError());
  const int64_t added = read_count(c, cnt);
  dt_append_dev(c, E, okey, oval, added);
  return added;
}

void dt_append_dev(Ctx* c, DEdges& E, const DBuf& key, const DBuf& val, int64_t na) {
  if (na == 0) return;
  cudaStream_t s = c->stream;
  DBuf k2, v2;
  k2.alloc(c, sizeof(uint64_t) * (E.m + na));
  v2.alloc(c, sizeof(uint64_t) * (E.m + na));
  if (E.m) {
    CUDA_OK(cudaMemcpyAsync(k2.p, E.key.p, sizeof(uint64_t) * E.m, cudaMemcpyDeviceToDevice, s));
    CUDA_OK(cudaMemcpyAsync(v2.p, E.val.p, sizeof(uint64_t) * E.m, cudaMemcpyDeviceToDevice, s));
  }
  CUDA_OK(cudaMemcpyAsync(k2.as<uint64_t>() + E.m, key.p, sizeof(uint64_t) * na, cudaMemcpyDeviceToDevice, s));
  CUDA_OK(cudaMemcpyAsync(v2.as<uint64_t>() + E.m, val.p, sizeof(uint64_t) * na, cudaMemcpyDeviceToDevice, s));
  std::swap(E.key, k2);
  std::swap(E.val, v2);
  E.m += na;
}

void dt_append(Ctx* c, DEdges& E, const std::vector<uint64_t>& key, const std::vector<uint64_t>& val) {
  DBuf k, v;
  upload(c, k, key.data(), (int64_t)key.size());
  upload(c, v, val.data(), (int64_t)val.size());
  dt_append_dev(c, E, k, v, (int64_t)key.size());
  CUDA_OK(cudaStreamSynchronize(c->stream));
}

void dt_logical(Ctx* c, const DEdges& E, const DBuf& s2o, int64_t n, DBuf& lp, DBuf& ld, DBuf& lw, DBuf* keys) {
  cudaStream_t s = c->stream;
  DBuf lkey, lval;
  lkey.alloc(c, sizeof(uint64_t) * std::max<int64_t>(E.m, 1));
  lval.alloc(c, sizeof(uint64_t) * std::max<int64_t>(E.m, 1));
  if (E.m)
    k_dt_logical<<<grid_for(c, E.m), 256, 0, s>>>(E.key.as<unsigned long long>(), E.val.as<unsigned long long>(), E.m,
                                                   s2o.as<int32_t>(), lkey.as<unsigned long long>(),
                                                   lval.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  sort_pairs(c, lkey, lval, E.m, 32 + slot_bits(n));
  DEdges L;
  L.m = E.m;
  std::swap(L.key, lkey);
  dt_row_ptr(c, L, n, lp);
  ld.alloc(c, sizeof(int32_t) * std::max<int64_t>(E.m, 1));
  lw.alloc(c, sizeof(uint32_t) * std::max<int64_t>(E.m, 1));
  if (E.m)
    k_dt_split<<<grid_for(c, E.m), 256, 0, s>>>(L.key.as<unsigned long long>(), lval.as<unsigned long long>(), E.m,
                                                 ld.as<int32_t>(), lw.as<uint32_t>(), nullptr);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));
  if (keys) std::swap(*keys, L.key);
}

void dt_pairs(Ctx* c, const DBuf& ld, const DBuf& lw, int64_t m, DBuf& out) {
  out.alloc(c, sizeof(uint64_t) * std::max<int64_t>(m, 1));
  if (m)
    k_dt_pairs<<<grid_for(c, m), 256, 0, c->stream>>>(ld.as<int32_t>(), lw.as<uint32_t>(), m,
                                                       out.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
}

int64_t dt_undirected(Ctx* c, int64_t n, const DBuf& lkey, int64_t ml, DBuf& np, DBuf& nc) {
  cudaStream_t s = c->stream;
  DEdges U;
  U.key.alloc(c, sizeof(uint64_t) * std::max<int64_t>(2 * ml, 1));
  DBuf k1, tmp, cnt;
  if (ml) k_dt_sym<<<grid_for(c, ml), 256, 0, s>>>(lkey.as<unsigned long long>(), ml, U.key.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  const int64_t m2 = 2 * ml;
  int64_t mu = 0;
  if (m2) {
    k1.alloc(c, sizeof(uint64_t) * m2);
    cub::DoubleBuffer<uint64_t> dk(U.key.as<uint64_t>(), k1.as<uint64_t>());
    size_t tb = 0;
    const int bits = 32 + slot_bits(n);
    CUDA_OK(cub::DeviceRadixSort::SortKeys(nullptr, tb, dk, m2, 0, bits, s));
    tmp.alloc(c, tb);
    CUDA_OK(cub::DeviceRadixSort::SortKeys(tmp.p, tb, dk, m2, 0, bits, s));
    uint64_t* sorted = dk.Current();
    uint64_t* other = sorted == U.key.as<uint64_t>() ? k1.as<uint64_t>() : U.key.as<uint64_t>();
    cnt.alloc(c, 8);
    size_t tu = 0;
    CUDA_OK(cub::DeviceSelect::Unique(nullptr, tu, sorted, other, cnt.as<int64_t>(), m2, s));
    tmp.alloc(c, tu);
    CUDA_OK(cub::DeviceSelect::Unique(tmp.p, tu, sorted, other, cnt.as<int64_t>(), m2, s));
    mu = read_count(c, cnt);
    if (other == k1.as<uint64_t>()) std::swap(U.key, k1);
  }
  U.m = mu;
  dt_row_ptr(c, U, n, np);
  nc.alloc(c, sizeof(int32_t) * std::max<int64_t>(mu, 1));
  if (mu)
    k_dt_split<<<grid_for(c, mu), 256, 0, s>>>(U.key.as<unsigned long long>(), U.key.as<unsigned long long>(), mu,
                                                nc.as<int32_t>(), nullptr, nullptr);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));
  return mu;
}

void dt_degnorm(Ctx* c, DEdges& E, int64_t ns, int64_t n, const std::vector<uint8_t>& kind, const DBuf& s2o,
                const std::vector<int32_t>& owner, int64_t th, int64_t f, bool combined, int rule,
                std::vector<int32_t>& sched, int64_t& added) {
  cudaStream_t s = c->stream;
  added = 0;
  // pre-§4 logical out adjacency (the padding's 2-hop candidates, R32)
  DBuf lp, ld, lw;
  dt_logical(c, E, s2o, n, lp, ld, lw, nullptr);
  dt_sort(c, E, ns);
  DBuf rp, dkind, order, tmp;
  dt_row_ptr(c, E, ns, rp);
  upload(c, dkind, kind.data(), ns);
  int64_t no = 0;
  order.alloc(c, sizeof(int32_t) * std::max<int64_t>(ns, 1));
  if (combined) {
    // combined mode (P@35029): no reorder, warps = 32-slot groups of the §2 layout
    launch_iota_i32(c, order.as<int32_t>(), ns);
    no = ns;
  } else if (ns) {
    // non-hole slots in id order, then a stable sort by bucket, descending
    DBuf idx, flag, cnt, bk0, bk1, ord1;
    idx.alloc(c, sizeof(int32_t) * ns);
    flag.alloc(c, ns);
    cnt.alloc(c, 8);
    k_dt_nonhole_flag<<<grid_for(c, ns), 256, 0, s>>>(dkind.as<uint8_t>(), ns, idx.as<int32_t>(), flag.as<uint8_t>());
    CUDA_OK(cudaGetLastError());
    size_t tb = 0;
    CUDA_OK(cub::DeviceSelect::Flagged(nullptr, tb, idx.as<int32_t>(), flag.as<uint8_t>(), order.as<int32_t>(),
                                       cnt.as<int64_t>(), ns, s));
    tmp.alloc(c, tb);
    CUDA_OK(cub::DeviceSelect::Flagged(tmp.p, tb, idx.as<int32_t>(), flag.as<uint8_t>(), order.as<int32_t>(),
                                       cnt.as<int64_t>(), ns, s));
    no = read_count(c, cnt);
    if (no) {
      bk0.alloc(c, sizeof(uint32_t) * no);
      bk1.alloc(c, sizeof(uint32_t) * no);
      ord1.alloc(c, sizeof(int32_t) * no);
      k_dt_bucket_key<<<grid_for(c, no), 256, 0, s>>>(rp.as<int64_t>(), order.as<int32_t>(), no, bk0.as<uint32_t>());
      CUDA_OK(cudaGetLastError());
      cub::DoubleBuffer<uint32_t> dk(bk0.as<uint32_t>(), bk1.as<uint32_t>());
      cub::DoubleBuffer<int32_t> dv(order.as<int32_t>(), ord1.as<int32_t>());
      CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, no, 0, 8, s));
      tmp.alloc(c, tb);
      CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, no, 0, 8, s));
      if (dv.Current() != order.as<int32_t>()) std::swap(order, ord1);
    }
  }
  // padded slots and their budgets
  DBuf qs, qu, qt, qcnt;
  qs.alloc(c, sizeof(int32_t) * std::max<int64_t>(no, 1));
  qu.alloc(c, sizeof(int32_t) * std::max<int64_t>(no, 1));
  qt.alloc(c, sizeof(int32_t) * std::max<int64_t>(no, 1));
  qcnt.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(qcnt.p, 0, 8, s));
  if (no)
    k_dt_pad_query<<<grid_for(c, no), 256, 0, s>>>(rp.as<int64_t>(), order.as<int32_t>(), no, dkind.as<uint8_t>(),
                                                   s2o.as<int32_t>(), th, f, qs.as<int32_t>(), qu.as<int32_t>(),
                                                   qt.as<int32_t>(), qcnt.as<unsigned long long>());
  CUDA_OK(cudaGetLastError());
  const int64_t nq = read_count(c, qcnt);
  sched.resize(no);
  if (no) CUDA_OK(cudaMemcpyAsync(sched.data(), order.p, sizeof(int32_t) * no, cudaMemcpyDeviceToHost, s));
  std::vector<int32_t> hqs(nq), hqt(nq);
  if (nq) {
    CUDA_OK(cudaMemcpyAsync(hqs.data(), qs.p, sizeof(int32_t) * nq, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaMemcpyAsync(hqt.data(), qt.p, sizeof(int32_t) * nq, cudaMemcpyDeviceToHost, s));
  }
  CUDA_OK(cudaStreamSynchronize(s));
  if (nq == 0) return;
  std::vector<int64_t> rptr;
  std::vector<uint64_t> rkeys;
  gpu_pad_candidates_dev(c, n, lp.as<int64_t>(), ld.as<int32_t>(), lw.as<uint32_t>(), nq, qu.as<int32_t>(),
                         hqt.data(), rule, rptr, rkeys);
  std::vector<uint64_t> ak, av;
  ak.reserve(rkeys.size());
  av.reserve(rkeys.size());
  for (int64_t i = 0; i < nq; i++)
    for (int64_t j = rptr[i]; j < rptr[i + 1]; j++) {
      const int32_t q = (int32_t)(rkeys[j] & 0xffffffffull);
      ak.push_back(((uint64_t)(uint32_t)hqs[i] << 32) | (uint32_t)owner[q]);
      av.push_back((rkeys[j] >> 32) | ((uint64_t)ADD_DEGNORM << 32));
    }
  added = (int64_t)ak.size();
  dt_append(c, E, ak, av);
}

void dt_export(Ctx* c, DEdges& E, int64_t ns, SlotGraph& out) {
  cudaStream_t s = c->stream;
  dt_sort(c, E, ns);
  DBuf rp, dst, w, add;
  dt_row_ptr(c, E, ns, rp);
  dst.alloc(c, sizeof(int32_t) * std::max<int64_t>(E.m, 1));
  w.alloc(c, sizeof(uint32_t) * std::max<int64_t>(E.m, 1));
  add.alloc(c, std::max<int64_t>(E.m, 1));
  if (E.m)
    k_dt_split<<<grid_for(c, E.m), 256, 0, s>>>(E.key.as<unsigned long long>(), E.val.as<unsigned long long>(), E.m,
                                                 dst.as<int32_t>(), w.as<uint32_t>(), add.as<uint8_t>());
  CUDA_OK(cudaGetLastError());
  E.key.reset();
  E.val.reset();
  out.rp.resize(ns + 1);
  out.col.resize(E.m);
  out.w.resize(E.m);
  out.added.resize(E.m);
  out.m_slots = E.m;
  CUDA_OK(cudaMemcpyAsync(out.rp.data(), rp.p, sizeof(int64_t) * (ns + 1), cudaMemcpyDeviceToHost, s));
  if (E.m) {
    CUDA_OK(cudaMemcpyAsync(out.col.data(), dst.p, sizeof(int32_t) * E.m, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaMemcpyAsync(out.w.data(), w.p, sizeof(uint32_t) * E.m, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaMemcpyAsync(out.added.data(), add.p, E.m, cudaMemcpyDeviceToHost, s));
  }
  CUDA_OK(cudaStreamSynchronize(s));
  E.m = 0;
}

}  // namespace gx
