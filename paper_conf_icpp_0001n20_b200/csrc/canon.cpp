// canon.cpp -- host canonicalisation of the uploaded CSR (SURVEY.md §8(a) A0,
// reading R2: the paper is silent on self-loops / duplicates).  Self-loops are
// dropped; a duplicate (u,v) is merged into its first occurrence's position
// and keeps the minimum weight; otherwise each row keeps the caller's order
// (the §2 cursor walks adjacency in input order, PAPER.md P@21936).
#include <omp.h>

#include <algorithm>

#include "gx_internal.h"

namespace gx {

namespace {
// Canonical row into (oc, ow); returns its length.  Small rows: quadratic
// scan; large rows: sort (col, pos) pairs.
int64_t canon_row(int64_t u, const int32_t* c, const uint32_t* w, int64_t d, int32_t* oc,
                  uint32_t* ow, std::vector<std::pair<int64_t, int64_t>>& tmp) {
  if (d <= 48) {
    int64_t k = 0;
    for (int64_t i = 0; i < d; i++) {
      int32_t v = c[i];
      uint32_t ww = w ? w[i] : 1u;
      if (v == (int32_t)u) continue;
      int64_t j = 0;
      for (; j < k; j++)
        if (oc[j] == v) break;
      if (j < k) {
        if (ww < ow[j]) ow[j] = ww;
      } else {
        oc[k] = v;
        ow[k] = ww;
        k++;
      }
    }
    return k;
  }
  tmp.clear();
  for (int64_t i = 0; i < d; i++)
    if (c[i] != (int32_t)u) tmp.push_back({(int64_t)c[i], i});
  std::sort(tmp.begin(), tmp.end());
  // first occurrence per destination, with its min weight
  std::vector<std::pair<int64_t, uint32_t>> keep;  // (pos, weight)
  keep.reserve(tmp.size());
  for (size_t i = 0; i < tmp.size();) {
    size_t j = i;
    uint32_t mw = 0xFFFFFFFFu;
    while (j < tmp.size() && tmp[j].first == tmp[i].first) {
      uint32_t ww = w ? w[tmp[j].second] : 1u;
      mw = std::min(mw, ww);
      j++;
    }
    keep.push_back({tmp[i].second, mw});
    i = j;
  }
  std::sort(keep.begin(), keep.end());
  for (size_t i = 0; i < keep.size(); i++) {
    oc[i] = c[keep[i].first];
    ow[i] = keep[i].second;
  }
  return (int64_t)keep.size();
}
}  // namespace

void canonicalize_host(int64_t n, const int64_t* rp, const int32_t* col, const uint32_t* w,
                       HostCSR& out) {
  out.n = n;
  out.rp.assign(n + 1, 0);
  std::vector<int64_t> len(n, 0);
  int64_t m_in = rp[n];
  std::vector<int32_t> tc(m_in);
  std::vector<uint32_t> tw(m_in);
#pragma omp parallel
  {
    std::vector<std::pair<int64_t, int64_t>> tmp;
#pragma omp for schedule(dynamic, 4096)
    for (int64_t u = 0; u < n; u++) {
      int64_t a = rp[u], d = rp[u + 1] - a;
      len[u] = canon_row(u, col + a, w ? w + a : nullptr, d, tc.data() + a, tw.data() + a, tmp);
    }
  }
  for (int64_t u = 0; u < n; u++) out.rp[u + 1] = out.rp[u] + len[u];
  out.m = out.rp[n];
  out.col.resize(out.m);
  out.w.resize(out.m);
#pragma omp parallel for schedule(static)
  for (int64_t u = 0; u < n; u++) {
    std::copy(tc.begin() + rp[u], tc.begin() + rp[u] + len[u], out.col.begin() + out.rp[u]);
    std::copy(tw.begin() + rp[u], tw.begin() + rp[u] + len[u], out.w.begin() + out.rp[u]);
  }
}

void ensure_host(gx_graph* g) {
  if (g->host_valid) return;
  HostCSR& h = g->host;
  h.n = g->n;
  h.m = g->m;
  h.rp.resize(g->n + 1);
  h.col.resize(g->m);
  h.w.resize(g->m);
  cudaStream_t s = g->ctx->stream;
  CUDA_OK(cudaMemcpyAsync(h.rp.data(), g->in_rp.p, sizeof(int64_t) * (g->n + 1), cudaMemcpyDeviceToHost, s));
  if (g->m) {
    CUDA_OK(cudaMemcpyAsync(h.col.data(), g->in_col.p, sizeof(int32_t) * g->m, cudaMemcpyDeviceToHost, s));
    CUDA_OK(cudaMemcpyAsync(h.w.data(), g->in_w.p, sizeof(uint32_t) * g->m, cudaMemcpyDeviceToHost, s));
  }
  CUDA_OK(cudaStreamSynchronize(s));
  g->host_valid = true;
}

}  // namespace gx
