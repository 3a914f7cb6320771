// gtransform.cu -- GPU-resident pieces of the Graffix preprocessing (SURVEY.md
// §8(f) N1).  The transforms stay host C++ where they are sequential (the §2
// cursor numbering, the §3 budgeted greedy insertion); the bulk-parallel
// steps they consume run here on the graph's device and return exactly the
// values the host code would compute (bit-exact, tests/test_gpu_transform.py).
//
//  * triangles per vertex of the undirected simple view U (§3, "the clustering
//    coefficient" P@29857: CC(v) = T(v) / (d(v)(d(v)-1)/2)), by the forward
//    algorithm: orient every edge of U from lower to higher (degree, id) rank,
//    then every triangle {u, v, w} is found exactly once as w in F(u) ∩ F(v)
//    for the edge u -> v, and credited to all three corners.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstring>
#include <vector>

#include "gx_internal.h"
#include "kernels_common.cuh"

namespace gx {

__device__ __forceinline__ bool rank_less(uint32_t da, int32_t a, uint32_t db, int32_t b) {
  return da < db || (da == db && a < b);
}

// forward out-degree of every vertex: neighbours of higher (degree, id) rank
__global__ void k_fwd_count(const int64_t* __restrict__ np, const int32_t* __restrict__ nc, int64_t n,
                            uint32_t* __restrict__ fc) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    const int64_t a = np[u], b = np[u + 1];
    const uint32_t du = (uint32_t)(b - a);
    uint32_t c = 0;
    for (int64_t e = a + lane; e < b; e += 32) {
      const int32_t v = nc[e];
      c += rank_less(du, (int32_t)u, (uint32_t)(np[v + 1] - np[v]), v) ? 1u : 0u;
    }
    c = __reduce_add_sync(FULL, c);
    if (lane == 0) fc[u] = c;
  }
}

// F(u) in ascending id order (the order of N(u)): warp ballot compaction
__global__ void k_fwd_fill(const int64_t* __restrict__ np, const int32_t* __restrict__ nc, int64_t n,
                           const uint64_t* __restrict__ fp, int32_t* __restrict__ fw) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    const int64_t a = np[u], b = np[u + 1];
    const uint32_t du = (uint32_t)(b - a);
    uint64_t o = fp[u];
    for (int64_t e0 = a; e0 < b; e0 += 32) {
      const int64_t e = e0 + lane;
      int32_t v = 0;
      bool f = false;
      if (e < b) {
        v = nc[e];
        f = rank_less(du, (int32_t)u, (uint32_t)(np[v + 1] - np[v]), v);
      }
      const unsigned m = __ballot_sync(FULL, f);
      if (f) fw[o + __popc(m & lanemask_lt())] = v;
      o += __popc(m);
    }
  }
}

// warp per vertex u: for every v in F(u), |F(u) ∩ F(v)| by binary search of
// the shorter list's elements in the longer one; each common w is a triangle
__global__ void k_tri(const uint64_t* __restrict__ fp, const int32_t* __restrict__ fw, int64_t n,
                      unsigned long long* __restrict__ T) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < n; u += nw) {
    const uint64_t ua = fp[u], ub = fp[u + 1];
    unsigned long long tu = 0;
    for (uint64_t k = ua; k < ub; k++) {
      const int32_t v = fw[k];
      const uint64_t va = fp[v], vb = fp[v + 1];
      // iterate the shorter list, search the longer
      const bool us = (ub - ua) <= (vb - va);
      const uint64_t sa = us ? ua : va, sb = us ? ub : vb, la = us ? va : ua, lb = us ? vb : ub;
      unsigned long long c = 0;
      for (uint64_t i = sa + lane; i < sb; i += 32) {
        const int32_t w = fw[i];
        uint64_t lo = la, hi = lb;
        while (lo < hi) {
          const uint64_t mid = (lo + hi) >> 1;
          if (fw[mid] < w) lo = mid + 1;
          else hi = mid;
        }
        if (lo < lb && fw[lo] == w) {
          c++;
          atomicAdd(&T[w], 1ull);
        }
      }
      c = __reduce_add_sync(FULL, (unsigned)c);
      if (lane == 0 && c) atomicAdd(&T[v], c);
      tu += c;
    }
    if (lane == 0 && tu) atomicAdd(&T[u], tu);
  }
}

// T[v] = triangles of U at v.  np/nc: U as CSR (rows sorted ascending, no
// self-loops, no duplicates), host arrays; T: host out [n].
void gpu_triangles(Ctx* c, int64_t n, const int64_t* np, const int32_t* nc, int64_t* T) {
  cudaStream_t s = c->stream;
  const int64_t mm = np[n];
  DBuf dnp, dnc, dT;
  dnp.alloc(c, sizeof(int64_t) * (n + 1));
  dnc.alloc(c, sizeof(int32_t) * std::max<int64_t>(mm, 1));
  CUDA_OK(cudaMemcpyAsync(dnp.p, np, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, s));
  if (mm) CUDA_OK(cudaMemcpyAsync(dnc.p, nc, sizeof(int32_t) * mm, cudaMemcpyHostToDevice, s));
  dT.alloc(c, sizeof(unsigned long long) * std::max<int64_t>(n, 1));
  gpu_triangles_dev(c, n, dnp.as<int64_t>(), dnc.as<int32_t>(), mm, dT.as<unsigned long long>());
  if (n) CUDA_OK(cudaMemcpyAsync(T, dT.p, sizeof(int64_t) * n, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
}

// device-resident form: U as device CSR (dnp [n+1], dnc [mm]); dT [n] out
void gpu_triangles_dev(Ctx* c, int64_t n, const int64_t* dnp, const int32_t* dnc, int64_t mm,
                       unsigned long long* dT) {
  cudaStream_t s = c->stream;
  (void)mm;
  DBuf fc, fp, fw, tmp;
  fc.alloc(c, sizeof(uint64_t) * (n + 1));
  CUDA_OK(cudaMemsetAsync(fc.p, 0, sizeof(uint64_t) * (n + 1), s));
  const int grid = c->num_sms * 16;
  k_fwd_count<<<grid, 256, 0, s>>>(dnp, dnc, n, fc.as<uint32_t>());
  CUDA_OK(cudaGetLastError());
  // u64 offsets of the forward lists (their total can exceed 2^32)
  fp.alloc(c, sizeof(uint64_t) * (n + 1));
  {
    size_t tb = 0;
    cub::TransformInputIterator<uint64_t, cub::CastOp<uint64_t>, const uint32_t*> in(fc.as<uint32_t>(),
                                                                                      cub::CastOp<uint64_t>());
    CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, in, fp.as<uint64_t>(), n + 1, s));
    tmp.alloc(c, tb);
    CUDA_OK(cub::DeviceScan::ExclusiveSum(tmp.p, tb, in, fp.as<uint64_t>(), n + 1, s));
  }
  uint64_t nf = 0;
  CUDA_OK(cudaMemcpyAsync(&nf, fp.as<uint64_t>() + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  fw.alloc(c, sizeof(int32_t) * std::max<uint64_t>(nf, 1));
  k_fwd_fill<<<grid, 256, 0, s>>>(dnp, dnc, n, fp.as<uint64_t>(), fw.as<int32_t>());
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaMemsetAsync(dT, 0, sizeof(unsigned long long) * std::max<int64_t>(n, 1), s));
  k_tri<<<grid, 256, 0, s>>>(fp.as<uint64_t>(), fw.as<int32_t>(), n, dT);
  CUDA_OK(cudaGetLastError());
  CUDA_OK(cudaStreamSynchronize(s));
}

}  // namespace gx

namespace gx {

// ---------------------------------------------------------------- §2 levels
// Level-synchronous BFS over the out-edges (warp per frontier vertex): the
// first visit of v claims level[v] = lv + 1 with a CAS and appends v to the
// next frontier (warp-aggregated append).  Levels are BFS distances, so they
// do not depend on the order of the claims.
__global__ void k_bfs_expand(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                             const int32_t* __restrict__ qin, int64_t qn, int32_t* __restrict__ level, int32_t lv,
                             int32_t* __restrict__ qout, unsigned long long* __restrict__ qcnt) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < qn; i += nw) {
    const int32_t u = qin[i];
    const int64_t a = rp[u], b = rp[u + 1];
    for (int64_t e0 = a; e0 < b; e0 += 32) {
      const int64_t e = e0 + lane;
      bool claim = false;
      int32_t v = 0;
      if (e < b) {
        v = col[e];
        claim = level[v] < 0 && atomicCAS(&level[v], -1, lv + 1) == -1;
      }
      const unsigned m = __ballot_sync(FULL, claim);
      if (m) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(qcnt, (unsigned long long)__popc(m));
        base = __shfl_sync(FULL, base, 0);
        if (claim) qout[base + __popc(m & lanemask_lt())] = v;
      }
    }
  }
}

__global__ void k_bfs_seed(const int32_t* __restrict__ src, int64_t ns, int32_t* __restrict__ level) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < ns; i += (int64_t)gridDim.x * blockDim.x)
    level[src[i]] = 0;
}

__global__ void k_neg_deg(const int64_t* __restrict__ rp, int64_t n, uint32_t* __restrict__ key,
                          int32_t* __restrict__ id) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    key[v] = ~(uint32_t)(rp[v + 1] - rp[v]);
    id[v] = (int32_t)v;
  }
}

namespace {
// multi-source BFS levels from the `ns` sources already in q0 (device); level
// must be all -1 except what this call seeds
void bfs_levels(Ctx* c, const int64_t* rp, const int32_t* col, int64_t n, DBuf& q0, DBuf& q1, int64_t ns,
                int32_t* level, DBuf& cnt) {
  cudaStream_t s = c->stream;
  k_bfs_seed<<<grid_for(c, ns), 256, 0, s>>>(q0.as<int32_t>(), ns, level);
  int64_t qn = ns;
  int32_t lv = 0;
  const int grid = c->num_sms * 16;
  while (qn > 0) {
    CUDA_OK(cudaMemsetAsync(cnt.p, 0, 8, s));
    k_bfs_expand<<<(int)std::min<int64_t>(grid, (qn + 7) / 8), 256, 0, s>>>(
        rp, col, q0.as<int32_t>(), qn, level, lv, q1.as<int32_t>(), cnt.as<unsigned long long>());
    CUDA_OK(cudaGetLastError());
    unsigned long long h = 0;
    CUDA_OK(cudaMemcpyAsync(&h, cnt.p, 8, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaStreamSynchronize(s));
    qn = (int64_t)h;
    std::swap(q0, q1);
    lv++;
  }
}
}  // namespace

// Alg 2 l.2-6 (readings R3-R5) with the bulk on the device: the source order
// (out-degree desc, id asc: a stable radix sort of complemented degrees), the
// reachability sweep of the first source (which covers the giant component),
// and the multi-source BFS levels; the host continues the source walk over
// the vertices the first sweep did not reach (a DFS that only enters
// unvisited vertices, as in the host transform).
void gpu_bfs_forest(Ctx* c, int64_t n, const int64_t* rp, const int32_t* col, std::vector<int32_t>& sources,
                    std::vector<int32_t>& level) {
  cudaStream_t s = c->stream;
  sources.clear();
  level.assign(n, -1);
  if (n == 0) return;
  const int64_t m = rp[n];
  DBuf drp, dcol, k0, k1, v0, v1, tmp, lev, q0, q1, cnt;
  drp.alloc(c, sizeof(int64_t) * (n + 1));
  dcol.alloc(c, sizeof(int32_t) * std::max<int64_t>(m, 1));
  CUDA_OK(cudaMemcpyAsync(drp.p, rp, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, s));
  if (m) CUDA_OK(cudaMemcpyAsync(dcol.p, col, sizeof(int32_t) * m, cudaMemcpyHostToDevice, s));
  // source order
  k0.alloc(c, sizeof(uint32_t) * n);
  k1.alloc(c, sizeof(uint32_t) * n);
  v0.alloc(c, sizeof(int32_t) * n);
  v1.alloc(c, sizeof(int32_t) * n);
  k_neg_deg<<<grid_for(c, n), 256, 0, s>>>(drp.as<int64_t>(), n, k0.as<uint32_t>(), v0.as<int32_t>());
  cub::DoubleBuffer<uint32_t> dk(k0.as<uint32_t>(), k1.as<uint32_t>());
  cub::DoubleBuffer<int32_t> dv(v0.as<int32_t>(), v1.as<int32_t>());
  size_t tb = 0;
  CUDA_OK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, n, 0, 32, s));
  tmp.alloc(c, tb);
  CUDA_OK(cub::DeviceRadixSort::SortPairs(tmp.p, tb, dk, dv, n, 0, 32, s));
  std::vector<int32_t> order(n);
  CUDA_OK(cudaMemcpyAsync(order.data(), dv.Current(), sizeof(int32_t) * n, cudaMemcpyDeviceToHost, s));
  // reachability of the first source
  lev.alloc(c, sizeof(int32_t) * n);
  q0.alloc(c, sizeof(int32_t) * n);
  q1.alloc(c, sizeof(int32_t) * n);
  cnt.alloc(c, 8);
  CUDA_OK(cudaMemsetAsync(lev.p, 0xff, sizeof(int32_t) * n, s));
  CUDA_OK(cudaStreamSynchronize(s));
  CUDA_OK(cudaMemcpyAsync(q0.p, order.data(), sizeof(int32_t), cudaMemcpyHostToDevice, s));
  bfs_levels(c, drp.as<int64_t>(), dcol.as<int32_t>(), n, q0, q1, 1, lev.as<int32_t>(), cnt);
  CUDA_OK(cudaMemcpyAsync(level.data(), lev.p, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  // the rest of the source walk (host): vis = reached so far
  std::vector<uint8_t> vis(n);
  for (int64_t v = 0; v < n; v++) vis[v] = level[v] >= 0;
  std::vector<int32_t> stack;
  sources.push_back(order[0]);
  for (int64_t i = 1; i < n; i++) {
    const int32_t r = order[i];
    if (vis[r]) continue;
    sources.push_back(r);
    vis[r] = 1;
    stack.push_back(r);
    while (!stack.empty()) {
      const int32_t u = stack.back();
      stack.pop_back();
      for (int64_t e = rp[u]; e < rp[u + 1]; e++) {
        const int32_t v = col[e];
        if (!vis[v]) {
          vis[v] = 1;
          stack.push_back(v);
        }
      }
    }
  }
  // multi-source BFS levels from every source
  CUDA_OK(cudaMemsetAsync(lev.p, 0xff, sizeof(int32_t) * n, s));
  CUDA_OK(cudaMemcpyAsync(q0.p, sources.data(), sizeof(int32_t) * sources.size(), cudaMemcpyHostToDevice, s));
  bfs_levels(c, drp.as<int64_t>(), dcol.as<int32_t>(), n, q0, q1, (int64_t)sources.size(), lev.as<int32_t>(), cnt);
  CUDA_OK(cudaMemcpyAsync(level.data(), lev.p, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
}

}  // namespace gx

namespace gx {

// ---------------------------------------------------------------- §4 padding
// Candidates of the degree normalisation (P@33654-35029, readings R32/R33):
// for a padded vertex u, the logical 2-hop out-neighbours q not in N+(u) and
// not u, each with its lightest combined weight, ordered by (weight, id); the
// first `take` of them become edges.  Two segmented radix sorts per batch of
// queries: (q, w) keys to keep each q's minimum, then (w, q) keys.
__device__ __forceinline__ uint32_t combine_w_dev(uint32_t w1, uint32_t w2, int rule) {
  if (rule == GX_W_MAX) return max(w1, w2);
  if (rule == GX_W_MEAN) return max(1u, (uint32_t)(((uint64_t)w1 + w2) / 2));
  return w1 + w2;
}

// upper bound of query i's candidates: sum of |N+(x)| over x in N+(u)
__global__ void k_pad_count(const int64_t* __restrict__ lp, const int32_t* __restrict__ ld,
                            const int32_t* __restrict__ qu, int64_t nq, uint64_t* __restrict__ cnt) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < nq; i += nw) {
    const int32_t u = qu[i];
    unsigned long long c = 0;
    for (int64_t e = lp[u] + lane; e < lp[u + 1]; e += 32) {
      const int32_t x = ld[e];
      c += (unsigned long long)(lp[x + 1] - lp[x]);
    }
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
    if (lane == 0) cnt[i] = c;
  }
}

// (q << 32 | w) per 2-hop path u -> x -> q; excluded q (u itself or an out-
// neighbour of u) become the sentinel ~0 (sorted last)
__global__ void k_pad_fill(const int64_t* __restrict__ lp, const int32_t* __restrict__ ld,
                           const uint32_t* __restrict__ lw, const int32_t* __restrict__ qu, int64_t nq,
                           const uint64_t* __restrict__ off, uint64_t base, int rule,
                           unsigned long long* __restrict__ keys) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < nq; i += nw) {
    const int32_t u = qu[i];
    const int64_t ua = lp[u], ub = lp[u + 1];
    uint64_t o = off[i] - base;
    for (int64_t ex = ua; ex < ub; ex++) {
      const int32_t x = ld[ex];
      const uint32_t w1 = lw[ex];
      const int64_t xa = lp[x], xb = lp[x + 1];
      for (int64_t eq = xa + lane; eq < xb; eq += 32) {
        const int32_t q = ld[eq];
        bool keep = q != u;
        if (keep) {   // q in N+(u)?  (rows sorted by destination)
          int64_t lo = ua, hi = ub;
          while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (ld[mid] < q) lo = mid + 1;
            else hi = mid;
          }
          keep = !(lo < ub && ld[lo] == q);
        }
        keys[o + (eq - xa)] = keep ? (((unsigned long long)(uint32_t)q << 32) | combine_w_dev(w1, lw[eq], rule))
                                   : ~0ull;
      }
      o += (uint64_t)(xb - xa);
    }
  }
}

// first (q, w) of each q -> (w << 32 | q); repeats and sentinels -> ~0
__global__ void k_pad_dedupe(const unsigned long long* __restrict__ in, unsigned long long* __restrict__ out,
                             const uint64_t* __restrict__ off, int64_t nq, uint64_t base) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < nq; i += nw) {
    const uint64_t a = off[i] - base, b = off[i + 1] - base;
    for (uint64_t j = a + lane; j < b; j += 32) {
      const unsigned long long k = in[j];
      const bool first = k != ~0ull && (j == a || (in[j - 1] >> 32) != (k >> 32));
      out[j] = first ? (((k & 0xffffffffull) << 32) | (k >> 32)) : ~0ull;
    }
  }
}

// the first take_i keys of every sorted segment (~0 where fewer exist)
__global__ void k_pad_take(const unsigned long long* __restrict__ k, const uint64_t* __restrict__ off, uint64_t base,
                           const int64_t* __restrict__ tptr, int64_t nq, unsigned long long* __restrict__ out) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const unsigned lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < nq; i += nw) {
    const uint64_t a = off[i] - base, len = off[i + 1] - off[i];
    const int64_t t0 = tptr[i], t = tptr[i + 1] - t0;
    for (int64_t j = lane; j < t; j += 32) out[t0 - tptr[0] + j] = (uint64_t)j < len ? k[a + j] : ~0ull;
  }
}

// queries (vertex qu[i], at most qtake[i] edges); lout = G_L out-adjacency as
// CSR sorted by destination (host).  Out: for query i the chosen (w << 32 | q)
// keys in [rptr[i], rptr[i+1]) of rkeys, in (weight, id) order.
void gpu_pad_candidates(Ctx* c, int64_t n, const int64_t* lp, const int32_t* ld, const uint32_t* lw, int64_t nq,
                        const int32_t* qu, const int32_t* qtake, int rule, std::vector<int64_t>& rptr,
                        std::vector<uint64_t>& rkeys) {
  cudaStream_t s = c->stream;
  rptr.assign(nq + 1, 0);
  rkeys.clear();
  if (nq == 0) return;
  const int64_t m = lp[n];
  DBuf dlp, dld, dlw, dqu;
  dlp.alloc(c, sizeof(int64_t) * (n + 1));
  dld.alloc(c, sizeof(int32_t) * std::max<int64_t>(m, 1));
  dlw.alloc(c, sizeof(uint32_t) * std::max<int64_t>(m, 1));
  dqu.alloc(c, sizeof(int32_t) * nq);
  CUDA_OK(cudaMemcpyAsync(dlp.p, lp, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, s));
  if (m) {
    CUDA_OK(cudaMemcpyAsync(dld.p, ld, sizeof(int32_t) * m, cudaMemcpyHostToDevice, s));
    CUDA_OK(cudaMemcpyAsync(dlw.p, lw, sizeof(uint32_t) * m, cudaMemcpyHostToDevice, s));
  }
  CUDA_OK(cudaMemcpyAsync(dqu.p, qu, sizeof(int32_t) * nq, cudaMemcpyHostToDevice, s));
  gpu_pad_candidates_dev(c, n, dlp.as<int64_t>(), dld.as<int32_t>(), dlw.as<uint32_t>(), nq, dqu.as<int32_t>(), qtake,
                         rule, rptr, rkeys);
}

// device-resident form: G_L as device CSR (dlp, dld, dlw), queries dqu on the
// device, their budgets qtake on the host
void gpu_pad_candidates_dev(Ctx* c, int64_t n, const int64_t* dlp_, const int32_t* dld_, const uint32_t* dlw_,
                            int64_t nq, const int32_t* dqu_, const int32_t* qtake, int rule,
                            std::vector<int64_t>& rptr, std::vector<uint64_t>& rkeys) {
  cudaStream_t s = c->stream;
  rptr.assign(nq + 1, 0);
  rkeys.clear();
  if (nq == 0) return;
  (void)n;
  DBuf cnt, off, tmp, k0, k1, sb, kout;
  cnt.alloc(c, sizeof(uint64_t) * (nq + 1));
  off.alloc(c, sizeof(uint64_t) * (nq + 1));
  CUDA_OK(cudaMemsetAsync(cnt.p, 0, sizeof(uint64_t) * (nq + 1), s));
  const int grid = c->num_sms * 16;
  k_pad_count<<<grid, 256, 0, s>>>(dlp_, dld_, dqu_, nq, cnt.as<uint64_t>());
  CUDA_OK(cudaGetLastError());
  size_t tb = 0;
  CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt.as<uint64_t>(), off.as<uint64_t>(), nq + 1, s));
  tmp.alloc(c, tb);
  CUDA_OK(cub::DeviceScan::ExclusiveSum(tmp.p, tb, cnt.as<uint64_t>(), off.as<uint64_t>(), nq + 1, s));
  // output slots per query: qtake[i] (the caller's upper bound)
  std::vector<int64_t> htp(nq + 1, 0);
  for (int64_t i = 0; i < nq; i++) htp[i + 1] = htp[i] + std::max<int32_t>(qtake[i], 0);
  DBuf dtp;
  dtp.alloc(c, sizeof(int64_t) * (nq + 1));
  CUDA_OK(cudaMemcpyAsync(dtp.p, htp.data(), sizeof(int64_t) * (nq + 1), cudaMemcpyHostToDevice, s));
  std::vector<uint64_t> hoff(nq + 1);
  CUDA_OK(cudaMemcpyAsync(hoff.data(), off.p, sizeof(uint64_t) * (nq + 1), cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  // batches of queries with at most B candidate keys (segmented sorts take int sizes)
  const uint64_t B = uint64_t(1) << 28;
  std::vector<uint64_t> hk;
  int64_t i0 = 0;
  while (i0 < nq) {
    int64_t i1 = i0 + 1;
    while (i1 < nq && hoff[i1 + 1] - hoff[i0] <= B) i1++;
    const uint64_t base = hoff[i0], tot = hoff[i1] - base;
    const int64_t bq = i1 - i0;
    k0.alloc(c, sizeof(uint64_t) * std::max<uint64_t>(tot, 1));
    k1.alloc(c, sizeof(uint64_t) * std::max<uint64_t>(tot, 1));
    sb.alloc(c, sizeof(int64_t) * (bq + 1));
    std::vector<int64_t> seg(bq + 1);
    for (int64_t i = 0; i <= bq; i++) seg[i] = (int64_t)(hoff[i0 + i] - base);
    CUDA_OK(cudaMemcpyAsync(sb.p, seg.data(), sizeof(int64_t) * (bq + 1), cudaMemcpyHostToDevice, s));
    if (tot) {
      k_pad_fill<<<grid, 256, 0, s>>>(dlp_, dld_, dlw_, dqu_ + i0,
                                      bq, off.as<uint64_t>() + i0, base, rule, k0.as<unsigned long long>());
      CUDA_OK(cudaGetLastError());
      size_t t1 = 0;
      const int64_t* b0 = sb.as<int64_t>();
      CUDA_OK(cub::DeviceSegmentedSort::SortKeys(nullptr, t1, k0.as<uint64_t>(), k1.as<uint64_t>(), (int)tot,
                                                 (int)bq, b0, b0 + 1, s));
      tmp.alloc(c, t1);
      CUDA_OK(cub::DeviceSegmentedSort::SortKeys(tmp.p, t1, k0.as<uint64_t>(), k1.as<uint64_t>(), (int)tot, (int)bq,
                                                 b0, b0 + 1, s));
      k_pad_dedupe<<<grid, 256, 0, s>>>(k1.as<unsigned long long>(), k0.as<unsigned long long>(),
                                        off.as<uint64_t>() + i0, bq, base);
      CUDA_OK(cudaGetLastError());
      CUDA_OK(cub::DeviceSegmentedSort::SortKeys(tmp.p, t1, k0.as<uint64_t>(), k1.as<uint64_t>(), (int)tot, (int)bq,
                                                 b0, b0 + 1, s));
      // only the first take_i keys of each segment travel back
      const int64_t nt = htp[i1] - htp[i0];
      kout.alloc(c, sizeof(uint64_t) * std::max<int64_t>(nt, 1));
      k_pad_take<<<grid, 256, 0, s>>>(k1.as<unsigned long long>(), off.as<uint64_t>() + i0, base,
                                      dtp.as<int64_t>() + i0, bq, kout.as<unsigned long long>());
      CUDA_OK(cudaGetLastError());
      hk.resize(nt);
      if (nt) CUDA_OK(cudaMemcpyAsync(hk.data(), kout.p, sizeof(uint64_t) * nt, cudaMemcpyDeviceToHost, s));
      CUDA_OK(cudaStreamSynchronize(s));
    }
    for (int64_t i = i0; i < i1; i++) {
      if (tot)
        for (int64_t j = htp[i] - htp[i0]; j < htp[i + 1] - htp[i0] && hk[j] != ~0ull; j++) rkeys.push_back(hk[j]);
      rptr[i + 1] = (int64_t)rkeys.size();
    }
    i0 = i1;
  }
}

}  // namespace gx
