// sell.cu -- SELL-32 slab layouts (built once per graph on the device).
//
// A SELL-32 slab stores the rows of 32 "lanes" column-major: entry j of lane
// l sits at slab[off + 32*j + l], padded with a sentinel to the longest row of
// the slice.  One warp-wide load then reads the j-th edge of 32 rows (128
// contiguous bytes), and each lane walks its own row with no per-edge
// bookkeeping.  Two users:
//   * the exact-mode PageRank pull (pagerank.cu): the in-edges of each window
//     of PRW rows, light rows sorted by in-degree inside the window so that a
//     slice holds rows of similar length (little padding); rows with more than
//     PR_HEAVY in-edges are reduced warp-per-row instead;
//   * the paper's thread-per-vertex mapping (tpv.cu): lanes = the §4 warp
//     schedule (P@33432) or the §2 slot order, where the Graffix transforms
//     decide how uniform the lane degrees are (degree normalisation, §4).
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdlib>

#include "gx_internal.h"
#include "kernels_common.cuh"
#include "sell.cuh"

namespace gx {

// ---- exact-mode PR windows: sort each window's light rows by in-degree ----
// One CTA per window; key = (class, -deg, local id) so that light rows come
// first by decreasing degree, then heavy rows.  Writes lane_row (padded to a
// multiple of 32 per window with -1), per-window light/heavy counts.
template <int WR>
__global__ void __launch_bounds__(1024) k_pr_window_sort(const uint32_t* __restrict__ crp, int64_t n,
                                                         int32_t* __restrict__ lane_tmp, int32_t* __restrict__ heavy_tmp,
                                                         int32_t* __restrict__ nlight, int32_t* __restrict__ nheavy,
                                                         uint32_t heavy_thr) {
  __shared__ uint32_t key[WR];
  const int64_t w = blockIdx.x;
  const int64_t base = w * WR;
  for (int i = threadIdx.x; i < WR; i += blockDim.x) {
    int64_t r = base + i;
    uint32_t k = 0xFFFFFFFFu;  // beyond n: sorts last
    if (r < n) {
      uint32_t d = crp[r + 1] - crp[r];
      uint32_t cls = d > heavy_thr ? 1u : 0u;
      uint32_t dd = d > heavy_thr ? 0u : (heavy_thr - d);
      k = (cls << 31) | (dd << 12) | (uint32_t)i;   // WR <= 4096, heavy_thr < 2^19
    }
    key[i] = k;
  }
  __syncthreads();
  // bitonic sort of WR keys
  for (int size = 2; size <= WR; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = threadIdx.x; i < WR / 2; i += blockDim.x) {
        int lo = 2 * i - (i & (stride - 1));
        int hi = lo + stride;
        bool up = ((lo & size) == 0);
        uint32_t a = key[lo], b = key[hi];
        if ((a > b) == up) {
          key[lo] = b;
          key[hi] = a;
        }
      }
      __syncthreads();
    }
  }
  __shared__ int s_nl, s_nh;
  if (threadIdx.x == 0) {
    s_nl = 0;
    s_nh = 0;
  }
  __syncthreads();
  for (int i = threadIdx.x; i < WR; i += blockDim.x) {
    uint32_t k = key[i];
    if (k == 0xFFFFFFFFu) continue;
    if (k >> 31) atomicAdd(&s_nh, 1);
    else atomicAdd(&s_nl, 1);
  }
  __syncthreads();
  const int nl = s_nl;
  for (int i = threadIdx.x; i < WR; i += blockDim.x) {
    uint32_t k = key[i];
    int32_t row = (k == 0xFFFFFFFFu) ? -1 : (int32_t)(base + (k & 0xFFFu));
    if (i < nl) lane_tmp[w * WR + i] = row;
    else if (k != 0xFFFFFFFFu) heavy_tmp[w * WR + (i - nl)] = row;
  }
  if (threadIdx.x == 0) {
    nlight[w] = nl;
    nheavy[w] = s_nh;
  }
}

// compact the per-window sorted rows into the padded lane array
__global__ void k_pr_window_lanes(const int32_t* __restrict__ lane_tmp, const int32_t* __restrict__ heavy_tmp,
                                  const int32_t* __restrict__ nlight, const int32_t* __restrict__ nheavy,
                                  const int64_t* __restrict__ lane_off, const int64_t* __restrict__ heavy_off,
                                  int64_t nwin, int wr, int32_t* __restrict__ lane_row, int32_t* __restrict__ heavy_row) {
  for (int64_t w = blockIdx.x; w < nwin; w += gridDim.x) {
    int nl = nlight[w], nh = nheavy[w];
    int64_t lo = lane_off[w], lp = lane_off[w + 1] - lo;
    for (int i = threadIdx.x; i < lp; i += blockDim.x) lane_row[lo + i] = i < nl ? lane_tmp[w * wr + i] : -1;
    for (int i = threadIdx.x; i < nh; i += blockDim.x) heavy_row[heavy_off[w] + i] = heavy_tmp[w * wr + i];
  }
}

// ---- generic SELL-32 fill ----
__global__ void k_sell_len(const uint32_t* __restrict__ rp, const int32_t* __restrict__ lane_row, int64_t nslices,
                           uint32_t* __restrict__ slice_len) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t s = warp; s < nslices; s += nw) {
    int32_t r = lane_row[s * 32 + lane_id()];
    uint32_t d = r >= 0 ? rp[r + 1] - rp[r] : 0u;
    d = warp_max_u32(d);
    if (lane_id() == 0) slice_len[s] = d;
  }
}

template <class T>
__global__ void k_sell_fill(const uint32_t* __restrict__ rp, const T* __restrict__ payload, const int32_t* __restrict__ lane_row,
                            const uint32_t* __restrict__ slice_len, const uint64_t* __restrict__ slice_off, int64_t nslices,
                            T sentinel, T* __restrict__ slab) {
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const unsigned lane = lane_id();
  for (int64_t s = warp; s < nslices; s += nw) {
    int32_t r = lane_row[s * 32 + lane];
    uint32_t a = r >= 0 ? rp[r] : 0u, d = r >= 0 ? rp[r + 1] - a : 0u;
    uint32_t L = slice_len[s];
    uint64_t off = slice_off[s];
    for (uint32_t j = 0; j < L; j++) slab[off + 32ull * j + lane] = j < d ? payload[a + j] : sentinel;
  }
}

__global__ void k_mul32(const uint32_t* __restrict__ in, uint64_t* __restrict__ out, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = 32ull * in[i];
}

static int64_t scan_u32_to_u64(Ctx* c, const uint32_t* in, uint64_t* out, int64_t n) {
  // exclusive scan of n values scaled by 32 into n+1 offsets
  cudaStream_t s = c->stream;
  DBuf tmp, in64;
  in64.alloc(c, sizeof(uint64_t) * (n + 1));
  k_mul32<<<grid_for(c, n + 1), 256, 0, s>>>(in, in64.as<uint64_t>(), n + 1);
  const uint64_t* it = in64.as<uint64_t>();
  size_t tb = 0;
  CUDA_OK(cub::DeviceScan::ExclusiveSum(nullptr, tb, it, out, n + 1, s));
  tmp.alloc(c, tb);
  CUDA_OK(cub::DeviceScan::ExclusiveSum(tmp.p, tb, it, out, n + 1, s));
  uint64_t tot = 0;
  CUDA_OK(cudaMemcpyAsync(&tot, out + n, 8, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  return (int64_t)tot;
}

// lane_row must have one extra trailing element so that the scan can read
// index nslices (its value is irrelevant: slice_len[nslices] is zeroed).
template <class T>
int64_t build_sell(Ctx* c, const uint32_t* rp, const T* payload, const int32_t* lane_row, int64_t nslices, T sentinel,
                   DBuf& slice_len, DBuf& slice_off, DBuf& slab) {
  cudaStream_t s = c->stream;
  slice_len.alloc(c, sizeof(uint32_t) * (nslices + 1));
  slice_off.alloc(c, sizeof(uint64_t) * (nslices + 1));
  CUDA_OK(cudaMemsetAsync(slice_len.p, 0, sizeof(uint32_t) * (nslices + 1), s));
  if (nslices) k_sell_len<<<grid_for(c, nslices * 32), 256, 0, s>>>(rp, lane_row, nslices, slice_len.as<uint32_t>());
  CUDA_OK(cudaGetLastError());
  int64_t tot = scan_u32_to_u64(c, slice_len.as<uint32_t>(), slice_off.as<uint64_t>(), nslices);
  slab.alloc(c, sizeof(T) * std::max<int64_t>(tot, 1));
  if (nslices)
    k_sell_fill<T><<<grid_for(c, nslices * 32), 256, 0, s>>>(rp, payload, lane_row, slice_len.as<uint32_t>(),
                                                            slice_off.as<uint64_t>(), nslices, sentinel, slab.as<T>());
  CUDA_OK(cudaGetLastError());
  return tot;
}

template int64_t build_sell<uint32_t>(Ctx*, const uint32_t*, const uint32_t*, const int32_t*, int64_t, uint32_t, DBuf&,
                                      DBuf&, DBuf&);
template int64_t build_sell<uint2>(Ctx*, const uint32_t*, const uint2*, const int32_t*, int64_t, uint2, DBuf&, DBuf&,
                                   DBuf&);

// Windowed degree-sorted SELL-32 (exact-mode PR pull over the CSC, SSSP dense
// push over the CSR).
template <class T>
void build_window_sell(Ctx* c, const uint32_t* rp, const T* payload, int64_t n, T sentinel, SellLayout& L) {
  cudaStream_t s = c->stream;
  const int64_t nwin = (n + PRW - 1) / PRW;
  L.nwin = nwin;
  DBuf lane_tmp, heavy_tmp, nl, nh;
  lane_tmp.alloc(c, sizeof(int32_t) * std::max<int64_t>(nwin * PRW, 1));
  heavy_tmp.alloc(c, sizeof(int32_t) * std::max<int64_t>(nwin * PRW, 1));
  nl.alloc(c, sizeof(int32_t) * (nwin + 1));
  nh.alloc(c, sizeof(int32_t) * (nwin + 1));
  uint32_t heavy_thr = PR_HEAVY;
  if (const char* e = getenv("GX_PR_HEAVY")) heavy_thr = (uint32_t)std::max(1, std::min(atoi(e), 1 << 18));
  if (nwin) k_pr_window_sort<PRW><<<nwin, 1024, 0, s>>>(rp, n, lane_tmp.as<int32_t>(), heavy_tmp.as<int32_t>(),
                                                        nl.as<int32_t>(), nh.as<int32_t>(), heavy_thr);
  CUDA_OK(cudaGetLastError());
  std::vector<int32_t> hnl(nwin), hnh(nwin);
  CUDA_OK(cudaMemcpyAsync(hnl.data(), nl.p, sizeof(int32_t) * nwin, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaMemcpyAsync(hnh.data(), nh.p, sizeof(int32_t) * nwin, cudaMemcpyDeviceToHost, s));
  CUDA_OK(cudaStreamSynchronize(s));
  std::vector<int64_t> loff(nwin + 1, 0), hoff(nwin + 1, 0), soff(nwin + 1, 0);
  for (int64_t w = 0; w < nwin; w++) {
    int64_t lp = (hnl[w] + 31) / 32 * 32;
    loff[w + 1] = loff[w] + lp;
    hoff[w + 1] = hoff[w] + hnh[w];
    soff[w + 1] = loff[w + 1] / 32;
  }
  L.nslices = loff[nwin] / 32;
  L.nheavy = hoff[nwin];
  DBuf dloff, dhoff;
  dloff.alloc(c, sizeof(int64_t) * (nwin + 1));
  dhoff.alloc(c, sizeof(int64_t) * (nwin + 1));
  CUDA_OK(cudaMemcpyAsync(dloff.p, loff.data(), sizeof(int64_t) * (nwin + 1), cudaMemcpyHostToDevice, s));
  CUDA_OK(cudaMemcpyAsync(dhoff.p, hoff.data(), sizeof(int64_t) * (nwin + 1), cudaMemcpyHostToDevice, s));
  L.lane_row.alloc(c, sizeof(int32_t) * (loff[nwin] + 32));
  L.heavy_row.alloc(c, sizeof(int32_t) * std::max<int64_t>(hoff[nwin], 1));
  L.win_slice.alloc(c, sizeof(int64_t) * (nwin + 1));
  L.win_heavy.alloc(c, sizeof(int64_t) * (nwin + 1));
  CUDA_OK(cudaMemcpyAsync(L.win_slice.p, soff.data(), sizeof(int64_t) * (nwin + 1), cudaMemcpyHostToDevice, s));
  CUDA_OK(cudaMemcpyAsync(L.win_heavy.p, hoff.data(), sizeof(int64_t) * (nwin + 1), cudaMemcpyHostToDevice, s));
  if (nwin)
    k_pr_window_lanes<<<grid_for(c, nwin * 256), 256, 0, s>>>(lane_tmp.as<int32_t>(), heavy_tmp.as<int32_t>(), nl.as<int32_t>(),
                                                              nh.as<int32_t>(), dloff.as<int64_t>(), dhoff.as<int64_t>(), nwin,
                                                              PRW, L.lane_row.as<int32_t>(), L.heavy_row.as<int32_t>());
  CUDA_OK(cudaGetLastError());
  L.slab_len = build_sell<T>(c, rp, payload, L.lane_row.as<int32_t>(), L.nslices, sentinel, L.slice_len, L.slice_off, L.slab);
  CUDA_OK(cudaStreamSynchronize(s));
}

template void build_window_sell<uint32_t>(Ctx*, const uint32_t*, const uint32_t*, int64_t, uint32_t, SellLayout&);
template void build_window_sell<uint2>(Ctx*, const uint32_t*, const uint2*, int64_t, uint2, SellLayout&);

}  // namespace gx
