// transform.cpp -- the three Graffix transforms on the host (SURVEY.md §8(a)
// A1-A3, A5-A6, A8-A9), producing the slot graph the sweeps run on.
//
//   §2 coalescing (Alg 2, PAPER.md P@16373-18419): BFS-forest levels, cursor
//      renumbering into an isomorph with k-aligned levels (holes), bounded
//      replication of well-connected (vertex, chunk) pairs into the holes.
//   §3 memory latency (P@29857-32416): clustering coefficient on the
//      undirected view, CC-raising sibling edges under a global budget, and
//      disjoint {c} + N(c) subgraphs processed t ~ 2*diam times in shared memory.
//   §4 divergence (P@33145-35029): degree buckets, warps in bucket order,
//      2-hop padding towards ceil(0.85 * warp max).
// Readings R1..R44 decide every tie;
// thresholds are compared in integer ppm.  The oracle (oracle/transform.py)
// implements the same readings independently; tests compare the exports.
#include <omp.h>
#include <parallel/algorithm>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <numeric>
#include <unordered_map>

#include "gx_internal.h"

namespace gx {
namespace {

// GX_TRANSFORM_TRACE=1: sub-phase times on stderr
struct PhaseTimer {
  bool on = getenv("GX_TRANSFORM_TRACE") != nullptr;
  std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
  void operator()(const char* name) {
    if (!on) return;
    auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "  %-22s %8.1f ms\n", name, std::chrono::duration<double, std::milli>(now - t).count());
    t = now;
  }
};

// Release a vector of per-vertex vectors in parallel: the transforms build
// ~10^8 small rows at RMAT-26, whose serial destruction took seconds per
// structure (profiles/r2/c5_full_all3_transform_trace.txt)
template <class T>
void par_free(std::vector<std::vector<T>>& v) {
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t i = 0; i < (int64_t)v.size(); i++) std::vector<T>().swap(v[i]);
  std::vector<std::vector<T>>().swap(v);
}

// Weight of an added edge standing for the 2-hop path with hop weights w1, w2
// (gx_knobs.added_weight_rule): the sum (P@34493, R17) or one of
// the "alternative" rules P@34692 allows.
uint32_t combine_w(uint32_t w1, uint32_t w2, int rule) {
  switch (rule) {
    case GX_W_MAX: return std::max(w1, w2);
    case GX_W_MEAN: return std::max<uint32_t>(1u, (uint32_t)(((uint64_t)w1 + w2) / 2));
    default: return w1 + w2;
  }
}

int64_t ppm(double x) { return (int64_t)std::floor(x * 1e6 + 0.5); }

struct Edge {
  int32_t dst;
  uint32_t w;
  uint8_t added;
};

// Working slot graph: one row vector per slot.
struct Work {
  int64_t n = 0, n_slots = 0;
  std::vector<std::vector<Edge>> rows;
  std::vector<int32_t> slot_to_orig;
  std::vector<uint8_t> kind;
  std::vector<int32_t> owner;  // orig -> owner slot
  int64_t n_holes = 0, n_repl = 0, added_coal = 0;
};

void identity(const HostCSR& g, Work& W) {
  W.n = g.n;
  W.n_slots = g.n;
  W.rows.assign(g.n, {});
  W.slot_to_orig.resize(g.n);
  W.kind.assign(g.n, OWNER);
  W.owner.resize(g.n);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < g.n; u++) {
    W.slot_to_orig[u] = (int32_t)u;
    W.owner[u] = (int32_t)u;
    auto& r = W.rows[u];
    r.reserve(g.rp[u + 1] - g.rp[u]);
    for (int64_t e = g.rp[u]; e < g.rp[u + 1]; e++) r.push_back({g.col[e], g.w[e], ADD_NONE});
  }
}

// ---------------------------------------------------------------- §2
// Alg 2 l.2-6 with R3-R5: sources in (out-degree desc, id asc) order, a source
// starts a reachability BFS if not yet visited; level = multi-source BFS
// distance from the source set.
void bfs_forest(const HostCSR& g, std::vector<int32_t>& sources, std::vector<int32_t>& level) {
  const int64_t n = g.n;
  std::vector<int32_t> order(n);
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
    return (g.rp[a + 1] - g.rp[a]) > (g.rp[b + 1] - g.rp[b]);
  });
  std::vector<uint8_t> vis(n, 0);
  std::vector<int32_t> stack;
  sources.clear();
  for (int32_t s : order) {
    if (vis[s]) continue;
    sources.push_back(s);
    vis[s] = 1;
    stack.push_back(s);
    while (!stack.empty()) {
      int32_t u = stack.back();
      stack.pop_back();
      for (int64_t e = g.rp[u]; e < g.rp[u + 1]; e++) {
        int32_t v = g.col[e];
        if (!vis[v]) {
          vis[v] = 1;
          stack.push_back(v);
        }
      }
    }
  }
  level.assign(n, -1);
  std::vector<int32_t> fr(sources), nx;
  for (int32_t s : sources) level[s] = 0;
  int32_t lv = 0;
  while (!fr.empty()) {
    nx.clear();
    for (int32_t u : fr)
      for (int64_t e = g.rp[u]; e < g.rp[u + 1]; e++) {
        int32_t v = g.col[e];
        if (level[v] < 0) {
          level[v] = lv + 1;
          nx.push_back(v);
        }
      }
    fr.swap(nx);
    lv++;
  }
}

// RenumberVertex (Alg 2 l.10-20), cursor reading R6-R8, pad R9.
void renumber(const HostCSR& g, int k, std::vector<int32_t>& nw, int64_t& n_slots,
              std::vector<std::pair<int64_t, int64_t>>& ranges, Ctx* dev) {
  const int64_t n = g.n;
  std::vector<int32_t> sources, level;
  PhaseTimer pt;
  if (dev) {
    gpu_bfs_forest(dev, n, g.rp.data(), g.col.data(), sources, level);   // N1 (gtransform.cu)
    pt("bfs_forest+levels (GPU)");
  } else {
    bfs_forest(g, sources, level);
    pt("bfs_forest+levels");
  }
  nw.assign(n, -1);
  // numbered[] mirrors nw[v] != -1 in one bit per vertex: the sequential
  // rounds below test it for every candidate child, and 8 MB stay in cache
  // where the 4-byte nw[] (268 MB at RMAT-26) does not
  std::vector<uint64_t> numbered((n + 63) / 64, 0);
  auto is_num = [&](int32_t v) { return (numbered[v >> 6] >> (v & 63)) & 1u; };
  auto set_num = [&](int32_t v) { numbered[v >> 6] |= 1ull << (v & 63); };
  for (size_t i = 0; i < sources.size(); i++) {
    nw[sources[i]] = (int32_t)i;
    set_num(sources[i]);
  }
  int64_t gid = (int64_t)sources.size();
  ranges.clear();
  ranges.push_back({0, gid});
  std::vector<int32_t> cur(sources), nxt;
  std::vector<int64_t> cursor, chp;
  std::vector<int32_t> ch;
  int32_t i = 0;
  while (true) {
    const int64_t start = (gid + k - 1) / k * k;
    std::vector<int32_t> parents(cur);
    // (nw values are unique: the parallel sort gives the sequential order)
    __gnu_parallel::sort(parents.begin(), parents.end(), [&](int32_t a, int32_t b) { return nw[a] < nw[b]; });
    // each parent's level-(i+1) neighbours in adjacency order, filtered in
    // parallel: level[] never changes during the numbering, so the cursor of
    // R6 walks exactly this list and skips the entries already numbered
    const int64_t np = (int64_t)parents.size();
    chp.assign(np + 1, 0);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t p = 0; p < np; p++) {
      const int32_t par = parents[p];
      int64_t cnt = 0;
      for (int64_t e = g.rp[par]; e < g.rp[par + 1]; e++) cnt += level[g.col[e]] == i + 1;
      chp[p + 1] = cnt;
    }
    for (int64_t p = 0; p < np; p++) chp[p + 1] += chp[p];
    ch.resize(chp[np]);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t p = 0; p < np; p++) {
      const int32_t par = parents[p];
      int64_t o = chp[p];
      for (int64_t e = g.rp[par]; e < g.rp[par + 1]; e++)
        if (level[g.col[e]] == i + 1) ch[o++] = g.col[e];
    }
    cursor.assign(chp.begin(), chp.end() - 1);
    nxt.clear();
    int64_t gid2 = start;
    // rounds: each parent numbers its next unnumbered level-(i+1) neighbour;
    // parents that exhausted their lists drop out of later rounds
    std::vector<size_t> live;
    live.reserve(np);
    for (int64_t p = 0; p < np; p++)
      if (chp[p + 1] > chp[p]) live.push_back((size_t)p);
    while (true) {
      bool assigned = false;
      size_t keep = 0;
      for (size_t li = 0; li < live.size(); li++) {
        const size_t p = live[li];
        int64_t c = cursor[p];
        const int64_t end = chp[p + 1];
        while (c < end && is_num(ch[c])) c++;
        if (c < end) {   // nxt[j] gets id start + j (written after the rounds, in parallel)
          gid2++;
          set_num(ch[c]);
          nxt.push_back(ch[c]);
          c++;
          assigned = true;
        }
        cursor[p] = c;
        if (c < end) live[keep++] = p;
      }
      live.resize(keep);
      if (!assigned) break;
    }
    // the level's ids: nw is not read inside the rounds (the numbered bits are),
    // so its random writes leave the sequential loop
    const int64_t nn = (int64_t)nxt.size();
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < nn; j++) nw[nxt[j]] = (int32_t)(start + j);
    if (nxt.empty()) break;
    ranges.push_back({start, gid2});
    gid = gid2;
    cur.swap(nxt);
    i++;
  }
  n_slots = n > 0 ? (gid + k - 1) / k * k : 0;
  pt("cursor numbering");
}

// Renumber + ReplicateVertex (Alg 2 l.21-35), readings R10-R18.
void coalesce(const HostCSR& g, int k, int64_t theta_ppm, int wrule, Work& W, Ctx* dev) {
  const int64_t n = g.n;
  std::vector<int32_t> nw;
  std::vector<std::pair<int64_t, int64_t>> ranges;
  int64_t n_slots = 0;
  renumber(g, k, nw, n_slots, ranges, dev);
  PhaseTimer pt;
  W.n = n;
  W.n_slots = n_slots;
  W.slot_to_orig.assign(n_slots, -1);
  W.kind.assign(n_slots, HOLE);
  W.owner = nw;
  for (int64_t u = 0; u < n; u++) {
    W.slot_to_orig[nw[u]] = (int32_t)u;
    W.kind[nw[u]] = OWNER;
  }
  // renumbered original adjacency (pre-move), CSR order
  std::vector<std::vector<Edge>> radj(n_slots);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) {
    auto& r = radj[nw[u]];
    r.reserve(g.rp[u + 1] - g.rp[u]);
    for (int64_t e = g.rp[u]; e < g.rp[u + 1]; e++) r.push_back({nw[g.col[e]], g.w[e], ADD_NONE});
  }
  pt("relabelled adjacency");
  std::vector<int32_t> nonhole((n_slots + k - 1) / k, 0);
  for (int64_t s = 0; s < n_slots; s++)
    if (W.kind[s] != HOLE) nonhole[s / k]++;
  // level of each chunk (levels are chunk-aligned from level 1 on)
  struct Asg {
    int32_t s;
    int64_t C;
    int64_t hole;
  };
  std::vector<Asg> asg;
  // chunk -> level index, for chunks of levels >= 1 whose previous level has holes
  const int64_t nchunks = (int64_t)nonhole.size();
  std::vector<int32_t> chunk_lv(nchunks, -1);
  for (size_t li = 1; li < ranges.size(); li++) {
    const int64_t holes = ranges[li].first - ranges[li - 1].second;
    if (holes <= 0) continue;
    for (int64_t C = ranges[li].first / k; C <= (ranges[li].second - 1) / k; C++) chunk_lv[C] = (int32_t)li;
  }
  // candidates (-count, s, C) per level: count the chunks of each row (rows
  // are short), in parallel over slots; since a level has h <= k-1 holes only
  // the h smallest candidates of each level matter, and the global h smallest
  // are among every thread's h smallest -- each thread keeps a bounded list
  using Cand = std::tuple<int64_t, int32_t, int64_t>;
  const size_t nlv = ranges.size();
  std::vector<int64_t> lv_holes(nlv, 0);
  for (size_t li = 1; li < nlv; li++) lv_holes[li] = std::max<int64_t>(0, ranges[li].first - ranges[li - 1].second);
  const int nth = omp_get_max_threads();
  std::vector<std::vector<std::vector<Cand>>> loc(nth, std::vector<std::vector<Cand>>(nlv));
#pragma omp parallel
  {
    auto& L = loc[omp_get_thread_num()];
    std::vector<int64_t> cs;
#pragma omp for schedule(dynamic, 4096)
    for (int64_t s = 0; s < n_slots; s++) {
      cs.clear();
      for (const Edge& e : radj[s]) {
        const int64_t C = e.dst / k;
        if (chunk_lv[C] >= 0) cs.push_back(C);
      }
      if (cs.empty()) continue;
      std::sort(cs.begin(), cs.end());
      for (size_t a = 0; a < cs.size();) {
        size_t b = a;
        while (b < cs.size() && cs[b] == cs[a]) b++;
        const int64_t cnt = (int64_t)(b - a), C = cs[a];
        a = b;
        if (cnt * 1000000 < theta_ppm * (int64_t)nonhole[C]) continue;
        auto& v = L[chunk_lv[C]];
        const size_t h = (size_t)lv_holes[chunk_lv[C]];
        const Cand c{-cnt, (int32_t)s, C};
        if (v.size() < h) {
          v.insert(std::upper_bound(v.begin(), v.end(), c), c);
        } else if (c < v.back()) {
          v.pop_back();
          v.insert(std::upper_bound(v.begin(), v.end(), c), c);
        }
      }
    }
  }
  pt("replica candidates");
  for (size_t li = 1; li < nlv; li++) {
    const int64_t h0 = ranges[li - 1].second, h1 = ranges[li].first;
    if (h1 <= h0) continue;
    std::vector<Cand> cl;
    for (int th = 0; th < nth; th++) cl.insert(cl.end(), loc[th][li].begin(), loc[th][li].end());
    std::sort(cl.begin(), cl.end());
    int64_t h = h0;
    for (auto& c : cl) {
      if (h >= h1) break;
      asg.push_back({std::get<1>(c), std::get<2>(c), h++});
    }
  }
  // replica rows from the pre-move rows (R16: 2-hop paths use n's pre-move
  // edges), then the owner rows take the renumbered rows by move -- no copy of
  // the whole adjacency -- and lose the moved edges
  int64_t added = 0;
  std::vector<std::vector<Edge>> rep_rows(asg.size());
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : added)
  for (size_t ai = 0; ai < asg.size(); ai++) {
    const Asg& a = asg[ai];
    const auto& orow = radj[a.s];
    std::vector<int32_t> nplus;
    nplus.reserve(orow.size());
    for (const Edge& e : orow) nplus.push_back(e.dst);
    std::sort(nplus.begin(), nplus.end());
    std::vector<Edge> row;
    for (const Edge& e : orow)
      if (e.dst / k == a.C) row.push_back(e);   // moved
    // 2-hop edges into chunk C with the minimum path weight (R16, R17)
    std::unordered_map<int32_t, uint32_t> best;
    for (const Edge& ev : orow)
      for (const Edge& eq : radj[ev.dst]) {
        const int32_t q = eq.dst;
        if (q / k != a.C || q == a.s || W.kind[q] == HOLE) continue;
        if (std::binary_search(nplus.begin(), nplus.end(), q)) continue;
        const uint32_t w = combine_w(ev.w, eq.w, wrule);
        auto it = best.find(q);
        if (it == best.end() || w < it->second) best[q] = w;
      }
    for (auto& kv : best) row.push_back({kv.first, kv.second, ADD_COALESCE});
    added += (int64_t)best.size();
    rep_rows[ai] = std::move(row);
  }
  W.rows = std::move(radj);
  for (size_t ai = 0; ai < asg.size(); ai++) {
    const Asg& a = asg[ai];
    auto& own = W.rows[a.s];
    own.erase(std::remove_if(own.begin(), own.end(), [&](const Edge& e) { return e.dst / k == a.C; }), own.end());
    W.rows[a.hole] = std::move(rep_rows[ai]);
    W.kind[a.hole] = REPLICA;
    W.slot_to_orig[a.hole] = W.slot_to_orig[a.s];
  }
  pt("replica rows");
  int64_t holes_left = 0;
  for (int64_t s = 0; s < n_slots; s++) holes_left += W.kind[s] == HOLE;
  W.n_repl = (int64_t)asg.size();
  W.n_holes = holes_left + W.n_repl;
  W.added_coal = added;
}

// ---------------------------------------------------------------- §3
// Mutable logical graph (original ids) with its undirected view U: flat CSR
// bases (built in one pass, or copied from the device) plus an overlay row per
// vertex the §3 insertion changed (<= 2 * budget of them), so no per-vertex
// containers are built or freed for the whole graph.
template <class T>
struct Span {
  const T* p = nullptr;
  size_t k = 0;
  Span() = default;
  Span(const T* p_, size_t k_) : p(p_), k(k_) {}
  Span(const std::vector<T>& v) : p(v.data()), k(v.size()) {}
  const T* begin() const { return p; }
  const T* end() const { return p + k; }
  size_t size() const { return k; }
  const T& operator[](size_t i) const { return p[i]; }
};
using OutE = std::pair<int32_t, uint32_t>;
struct Logical {
  int64_t n = 0;
  std::vector<int64_t> op, np;   // row offsets of the bases [n + 1]
  std::vector<OutE> oe;          // G_L out-edges (dst, w), rows sorted by dst
  std::vector<int32_t> ne;       // U neighbours, rows sorted ascending
  std::vector<int32_t> ovo, ovn; // vertex -> overlay row, or -1 (the base row)
  std::vector<std::vector<OutE>> xo;
  std::vector<std::vector<int32_t>> xn;
  std::vector<int64_t> T;        // triangles at each vertex

  void init_overlays() {
    ovo.assign(n, -1);
    ovn.assign(n, -1);
  }
  Span<OutE> out(int32_t a) const {
    const int32_t i = ovo[a];
    return i < 0 ? Span<OutE>(oe.data() + op[a], (size_t)(op[a + 1] - op[a])) : Span<OutE>(xo[i]);
  }
  Span<int32_t> N(int32_t c) const {
    const int32_t i = ovn[c];
    return i < 0 ? Span<int32_t>(ne.data() + np[c], (size_t)(np[c + 1] - np[c])) : Span<int32_t>(xn[i]);
  }
  std::vector<OutE>& out_mut(int32_t a) {
    if (ovo[a] < 0) {
      const Span<OutE> b = out(a);
      ovo[a] = (int32_t)xo.size();
      xo.emplace_back(b.begin(), b.end());
    }
    return xo[ovo[a]];
  }
  std::vector<int32_t>& N_mut(int32_t c) {
    if (ovn[c] < 0) {
      const Span<int32_t> b = N(c);
      ovn[c] = (int32_t)xn.size();
      xn.emplace_back(b.begin(), b.end());
    }
    return xn[ovn[c]];
  }

  int64_t d(int32_t c) const { return (int64_t)N(c).size(); }
  int64_t P(int32_t c) const { int64_t x = d(c); return x * (x - 1) / 2; }
  bool high(int32_t c, int64_t th) const { return (__int128)T[c] * 1000000 > (__int128)th * P(c); }
  bool adj(int32_t a, int32_t b) const { const auto r = N(a); return std::binary_search(r.begin(), r.end(), b); }
  const uint32_t* outw(int32_t a, int32_t b) const {
    const auto r = out(a);
    auto it = std::lower_bound(r.begin(), r.end(), std::make_pair(b, 0u),
                               [](const OutE& x, const OutE& y) { return x.first < y.first; });
    return (it != r.end() && it->first == b) ? &it->second : nullptr;
  }
  // sibling edge a->b for centre c: along a directed 2-path (R23), or any two
  // U-neighbours of c with the undirected variant (N3, P@29950)
  bool eligible(int32_t c, int32_t a, int32_t b, bool und) const {
    return und ? (adj(c, a) && adj(c, b)) : (outw(a, c) && outw(c, b));
  }
  // weight of the pair {a, b} in U: the lighter existing direction
  uint32_t wU(int32_t a, int32_t b) const {
    const uint32_t* x = outw(a, b);
    const uint32_t* y = outw(b, a);
    return x && y ? std::min(*x, *y) : (x ? *x : *y);
  }
  // |x ∩ y| of two sorted lists; f(v) for every common v.  A hub's list is
  // 10^5 long on RMAT, so a short list is searched into a long one
  // (O(|x| log |y|)) instead of merged (O(|x| + |y|)): the same set
  template <class F>
  static int64_t common(Span<int32_t> x, Span<int32_t> y, F&& f) {
    if (x.size() > y.size()) std::swap(x, y);
    int64_t r = 0;
    if (x.size() * 16 < y.size()) {
      const int32_t* lo = y.begin();
      for (int32_t v : x) {
        lo = std::lower_bound(lo, y.end(), v);
        if (lo == y.end()) break;
        if (*lo == v) { f(v); r++; }
      }
      return r;
    }
    size_t i = 0, j = 0;
    while (i < x.size() && j < y.size()) {
      if (x[i] < y[j]) i++;
      else if (x[i] > y[j]) j++;
      else { f(x[i]); r++; i++; j++; }
    }
    return r;
  }
  static int64_t inter(Span<int32_t> x, Span<int32_t> y) { return common(x, y, [](int32_t) {}); }
  void link(int32_t a, int32_t b, uint32_t w) {
    const bool fresh = !adj(a, b);
    auto& r = out_mut(a);
    auto it = std::lower_bound(r.begin(), r.end(), std::make_pair(b, 0u),
                               [](const OutE& x, const OutE& y) { return x.first < y.first; });
    r.insert(it, {b, w});
    if (fresh) {
      // common neighbours gain a triangle; a and b gain |common| each
      const int64_t cnt = common(N(a), N(b), [&](int32_t v) { T[v]++; });
      T[a] += cnt;
      T[b] += cnt;
      auto& na = N_mut(a);
      na.insert(std::lower_bound(na.begin(), na.end(), b), b);
      auto& nb = N_mut(b);
      nb.insert(std::lower_bound(nb.begin(), nb.end(), a), a);
    }
  }
};

// G_L out-adjacency (original ids, sorted by destination): the owner slot's
// row of every vertex in parallel, then the replica rows appended
void logical_out(const Work& W, std::vector<std::vector<std::pair<int32_t, uint32_t>>>& out) {
  const int64_t n = W.n;
  out.assign(n, {});
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) {
    const auto& row = W.rows[W.owner[u]];
    auto& r = out[u];
    r.reserve(row.size());
    for (const Edge& e : row) r.push_back({W.slot_to_orig[e.dst], e.w});
  }
  for (int64_t s = 0; s < W.n_slots; s++) {
    if (W.kind[s] != REPLICA) continue;
    auto& r = out[W.slot_to_orig[s]];
    for (const Edge& e : W.rows[s]) r.push_back({W.slot_to_orig[e.dst], e.w});
  }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) std::sort(out[u].begin(), out[u].end());
}

void build_logical(const Work& W, Logical& L, Ctx* dev) {
  PhaseTimer pt;
  const int64_t n = W.n;
  L.n = n;
  {
    std::vector<std::vector<OutE>> out;
    logical_out(W, out);
    L.op.assign(n + 1, 0);
    for (int64_t u = 0; u < n; u++) L.op[u + 1] = L.op[u] + (int64_t)out[u].size();
    L.oe.resize(L.op[n]);
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < n; u++) std::copy(out[u].begin(), out[u].end(), L.oe.begin() + L.op[u]);
    par_free(out);
  }
  // in-adjacency by counting (CSC of G_L)
  std::vector<int64_t> ip(n + 1, 0);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t e = 0; e < L.op[n]; e++) __atomic_fetch_add(&ip[L.oe[e].first + 1], 1, __ATOMIC_RELAXED);
  for (int64_t v = 0; v < n; v++) ip[v + 1] += ip[v];
  std::vector<int32_t> isrc(ip[n]);
  std::vector<int64_t> cur(ip.begin(), ip.end() - 1);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++)
    for (int64_t e = L.op[u]; e < L.op[u + 1]; e++)
      isrc[__atomic_fetch_add(&cur[L.oe[e].first], 1, __ATOMIC_RELAXED)] = (int32_t)u;
  pt("logical out+in");
  // U: sorted union of out- and in-neighbours, counted then filled
  std::vector<int64_t> cnt(n + 1, 0);
  std::vector<std::vector<int32_t>> tmp(omp_get_max_threads());
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) {
    auto& v = tmp[omp_get_thread_num()];
    v.clear();
    for (int64_t e = L.op[u]; e < L.op[u + 1]; e++) v.push_back(L.oe[e].first);
    for (int64_t i = ip[u]; i < ip[u + 1]; i++) v.push_back(isrc[i]);
    std::sort(v.begin(), v.end());
    cnt[u + 1] = (int64_t)(std::unique(v.begin(), v.end()) - v.begin());
  }
  L.np.assign(n + 1, 0);
  for (int64_t u = 0; u < n; u++) L.np[u + 1] = L.np[u] + cnt[u + 1];
  L.ne.resize(L.np[n]);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) {
    auto& v = tmp[omp_get_thread_num()];
    v.clear();
    for (int64_t e = L.op[u]; e < L.op[u + 1]; e++) v.push_back(L.oe[e].first);
    for (int64_t i = ip[u]; i < ip[u + 1]; i++) v.push_back(isrc[i]);
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
    std::copy(v.begin(), v.end(), L.ne.begin() + L.np[u]);
  }
  L.init_overlays();
  pt("undirected N");
  if (dev) {
    // N1: the forward-algorithm triangle count on the graph's device
    L.T.assign(n, 0);
    std::vector<int32_t> nc(L.ne);
    if (nc.empty()) nc.push_back(0);
    gpu_triangles(dev, n, L.np.data(), nc.data(), L.T.data());
    pt("triangles (GPU)");
    return;
  }
  // triangles: forward algorithm over the degree-ordered orientation
  L.T.assign(n, 0);
  std::vector<std::vector<int32_t>> fwd(n);
  auto rank_less = [&](int32_t a, int32_t b) {
    return L.d(a) < L.d(b) || (L.d(a) == L.d(b) && a < b);
  };
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; u++) {
    for (int32_t v : L.N((int32_t)u))
      if (rank_less((int32_t)u, v)) fwd[u].push_back(v);
    std::sort(fwd[u].begin(), fwd[u].end());
  }
  pt("forward lists");
  std::vector<int64_t> tl(n, 0);
#pragma omp parallel
  {
#pragma omp for schedule(dynamic, 1024)
    for (int64_t u = 0; u < n; u++) {
      for (int32_t v : fwd[u]) {
        const auto &x = fwd[u], &y = fwd[v];
        size_t i = 0, j = 0;
        while (i < x.size() && j < y.size()) {
          if (x[i] < y[j]) i++;
          else if (x[i] > y[j]) j++;
          else {
            const int32_t w = x[i];
#pragma omp atomic
            tl[u]++;
#pragma omp atomic
            tl[v]++;
#pragma omp atomic
            tl[w]++;
            i++;
            j++;
          }
        }
      }
    }
  }
  L.T.swap(tl);
  pt("triangles");
}

struct SmemOut {
  std::vector<std::tuple<int32_t, int32_t, uint32_t>> added;
  std::vector<std::tuple<int32_t, std::vector<int32_t>, int32_t>> tiles;
};

// The ids c in [0, n) with pred(c), ascending, collected in parallel (each
// thread a contiguous static range; the ranges are concatenated in order)
template <class T, class Pred, class Make>
std::vector<T> par_filter(int64_t n, Pred pred, Make make) {
  const int nt = omp_get_max_threads();
  std::vector<std::vector<T>> loc(nt);
#pragma omp parallel num_threads(nt)
  {
    const int t = omp_get_thread_num();
    const int64_t a = n * t / nt, b = n * (t + 1) / nt;
    for (int64_t c = a; c < b; c++)
      if (pred((int32_t)c)) loc[t].push_back(make((int32_t)c));
  }
  size_t tot = 0;
  for (auto& v : loc) tot += v.size();
  std::vector<T> out;
  out.reserve(tot);
  for (auto& v : loc) out.insert(out.end(), v.begin(), v.end());
  return out;
}

// CC edge insertion: case 1 (R22) then case 2 (R24, R25); budget in directed edges (R26)
void cc_edges(Logical& L, int64_t th, int64_t budget, int wrule, bool und, SmemOut& out) {
  PhaseTimer pt;
  const int64_t n = L.n;
  int64_t rem = budget;
  auto linkable = [&](int32_t c, int32_t a, int32_t b) {
    return !L.adj(a, b) && (L.eligible(c, a, b, und) || L.eligible(c, b, a, und));
  };
  auto do_link = [&](int32_t c, int32_t a, int32_t b) {
    const int32_t xs[2] = {a, b}, ys[2] = {b, a};
    for (int q = 0; q < 2; q++) {
      if (rem <= 0) return;
      const int32_t x = xs[q], y = ys[q];
      if (L.eligible(c, x, y, und) && !L.outw(x, y)) {
        const uint32_t w = und ? combine_w(L.wU(x, c), L.wU(c, y), wrule) : combine_w(*L.outw(x, c), *L.outw(c, y), wrule);
        L.link(x, y, w);
        out.added.push_back({x, y, w});
        rem--;
      }
    }
  };
  // case 1
  // (keys are unique: the parallel sort gives the sequential order)
  std::vector<std::pair<int64_t, int32_t>> cands = par_filter<std::pair<int64_t, int32_t>>(
      n, [&](int32_t c) { return L.d(c) >= 2 && !L.high(c, th); },
      [&](int32_t c) {
        return std::make_pair((int64_t)(((__int128)th * L.P(c)) / 1000000) + 1 - L.T[c], c);
      });
  __gnu_parallel::sort(cands.begin(), cands.end());
  pt("case-1 centres");
  for (auto& cn : cands) {
    if (rem <= 0) break;
    const int32_t c = cn.second;
    const int64_t P = L.P(c);
    const int64_t need = (int64_t)(((__int128)th * P) / 1000000) + 1 - L.T[c];
    if (need <= 0) continue;
    if (P - L.T[c] < need) continue;
    const Span<int32_t> nsp = L.N(c);
    const std::vector<int32_t> Nc(nsp.begin(), nsp.end());
    std::vector<std::tuple<int64_t, int32_t, int32_t>> pairs;
    for (size_t i = 0; i < Nc.size(); i++)
      for (size_t j = i + 1; j < Nc.size(); j++) {
        const int32_t a = Nc[i], b = Nc[j];
        if (linkable(c, a, b)) pairs.push_back({-Logical::inter(L.N(a), L.N(b)), a, b});
      }
    if ((int64_t)pairs.size() < need) continue;
    std::sort(pairs.begin(), pairs.end());
    for (auto& p : pairs) {
      if (rem <= 0 || L.high(c, th)) break;
      const int32_t a = std::get<1>(p), b = std::get<2>(p);
      if (linkable(c, a, b)) do_link(c, a, b);
    }
  }
  pt("case 1");
  // case 2
  if (rem > 0) {
    std::vector<int32_t> highs =
        par_filter<int32_t>(n, [&](int32_t c) { return L.high(c, th); }, [](int32_t c) { return c; });
    __gnu_parallel::sort(highs.begin(), highs.end(), [&](int32_t x, int32_t y) {
      const __int128 lhs = (__int128)L.T[x] * L.P(y), rhs = (__int128)L.T[y] * L.P(x);
      if (lhs != rhs) return lhs > rhs;
      return x < y;
    });
    while (rem > 0) {
      bool any = false;
      for (int32_t c : highs) {
        if (rem <= 0) break;
        const Span<int32_t> nsp = L.N(c);
        const std::vector<int32_t> Nc(nsp.begin(), nsp.end());
        std::unordered_map<int32_t, int64_t> intdeg;
        for (int32_t a : Nc) intdeg[a] = Logical::inter(L.N(a), Nc);
        std::vector<int32_t> sib(Nc);
        std::sort(sib.begin(), sib.end(), [&](int32_t x, int32_t y) {
          return intdeg[x] != intdeg[y] ? intdeg[x] < intdeg[y] : x < y;
        });
        bool done = false;
        for (int32_t a : sib) {
          int32_t best = -1;
          for (int32_t b : Nc) {
            if (b == a || !linkable(c, a, b)) continue;
            if (best < 0 || intdeg[b] < intdeg[best] || (intdeg[b] == intdeg[best] && b < best)) best = b;
          }
          if (best >= 0) {
            do_link(c, std::min(a, best), std::max(a, best));
            done = true;
            break;
          }
        }
        any |= done;
      }
      if (!any) break;
    }
  }
}

// disjoint shared-memory subgraphs (R27, R28)
void subgraphs(const Logical& L, int64_t th, int smax, int smem_iters, SmemOut& out) {
  const int64_t n = L.n;
  std::vector<int32_t> cs = par_filter<int32_t>(
      n, [&](int32_t c) { return L.high(c, th) && 1 + L.d(c) <= smax; }, [](int32_t c) { return c; });
  __gnu_parallel::sort(cs.begin(), cs.end(), [&](int32_t x, int32_t y) {
    const __int128 lhs = (__int128)L.T[x] * L.P(y), rhs = (__int128)L.T[y] * L.P(x);
    if (lhs != rhs) return lhs > rhs;
    if (L.d(x) != L.d(y)) return L.d(x) > L.d(y);
    return x < y;
  });
  std::vector<uint8_t> used(n, 0);
  for (int32_t c : cs) {
    bool free = !used[c];
    const Span<int32_t> nsp = L.N(c);
    for (int32_t v : nsp) free = free && !used[v];
    if (!free) continue;
    std::vector<int32_t> S(nsp.begin(), nsp.end());
    S.push_back(c);
    std::sort(S.begin(), S.end());
    for (int32_t v : S) used[v] = 1;
    const int64_t d = L.d(c);
    const bool clique = L.T[c] == d * (d - 1) / 2;
    const int32_t t = smem_iters > 0 ? smem_iters : 2 * (clique ? 1 : 2);
    out.tiles.push_back({c, std::move(S), t});
  }
}

// ---------------------------------------------------------------- §4
int bucket_of(int64_t d) {
  int b = 0;
  while (d) {
    b++;
    d >>= 1;
  }
  return b;  // R30: 0 for d = 0, else 1 + floor(log2 d)
}

void degnorm(Work& W, int64_t th, int64_t f, bool combined, int wrule, std::vector<int32_t>& sched, int64_t& added,
             Ctx* dev) {
  PhaseTimer pt;
  const int64_t ns = W.n_slots;
  std::vector<int64_t> deg(ns);
  for (int64_t s = 0; s < ns; s++) deg[s] = (int64_t)W.rows[s].size();
  std::vector<int32_t> order;
  if (combined) {
    order.resize(ns);
    std::iota(order.begin(), order.end(), 0);
  } else {
    for (int64_t s = 0; s < ns; s++)
      if (W.kind[s] != HOLE) order.push_back((int32_t)s);
    std::stable_sort(order.begin(), order.end(),
                     [&](int32_t a, int32_t b) { return bucket_of(deg[a]) > bucket_of(deg[b]); });
  }
  // pre-§4 logical out adjacency
  std::vector<std::vector<std::pair<int32_t, uint32_t>>> lout;
  logical_out(W, lout);
  pt("order + logical out");
  std::vector<std::vector<Edge>> adds(ns);
  const int64_t nwarps = ((int64_t)order.size() + 31) / 32;
  if (dev) {
    // N1: the padded slots are found here (per-warp M and target), their
    // candidates ranked on the device (gtransform.cu gpu_pad_candidates)
    std::vector<int32_t> qs, qu, qtake;
    for (int64_t wi = 0; wi < nwarps; wi++) {
      const int64_t b0 = wi * 32, b1 = std::min<int64_t>(b0 + 32, (int64_t)order.size());
      int64_t M = 0;
      for (int64_t i = b0; i < b1; i++) M = std::max(M, deg[order[i]]);
      const int64_t target = (f * M + 999999) / 1000000;
      for (int64_t i = b0; i < b1; i++) {
        const int32_t s = order[i];
        const int64_t d = deg[s];
        if (W.kind[s] != OWNER || !(0 < d && d < M)) continue;
        if (!((M - d) * 1000000 < th * M)) continue;
        if (d >= target) continue;
        qs.push_back(s);
        qu.push_back(W.slot_to_orig[s]);
        qtake.push_back((int32_t)(target - d));
      }
    }
    std::vector<int64_t> lp(W.n + 1, 0);
    for (int64_t u = 0; u < W.n; u++) lp[u + 1] = lp[u] + (int64_t)lout[u].size();
    std::vector<int32_t> ld(std::max<int64_t>(lp[W.n], 1));
    std::vector<uint32_t> lw(std::max<int64_t>(lp[W.n], 1));
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < W.n; u++)
      for (size_t j = 0; j < lout[u].size(); j++) {
        ld[lp[u] + j] = lout[u][j].first;
        lw[lp[u] + j] = lout[u][j].second;
      }
    std::vector<int64_t> rptr;
    std::vector<uint64_t> rkeys;
    gpu_pad_candidates(dev, W.n, lp.data(), ld.data(), lw.data(), (int64_t)qs.size(), qu.data(), qtake.data(), wrule,
                       rptr, rkeys);
    for (size_t i = 0; i < qs.size(); i++)
      for (int64_t j = rptr[i]; j < rptr[i + 1]; j++)
        adds[qs[i]].push_back({W.owner[(int32_t)(rkeys[j] & 0xffffffffull)], (uint32_t)(rkeys[j] >> 32), ADD_DEGNORM});
    pt("padding candidates (GPU)");
  } else {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t wi = 0; wi < nwarps; wi++) {
    const int64_t b0 = wi * 32, b1 = std::min<int64_t>(b0 + 32, (int64_t)order.size());
    int64_t M = 0;
    for (int64_t i = b0; i < b1; i++) M = std::max(M, deg[order[i]]);
    const int64_t target = (f * M + 999999) / 1000000;
    for (int64_t i = b0; i < b1; i++) {
      const int32_t s = order[i];
      const int64_t d = deg[s];
      if (W.kind[s] != OWNER || !(0 < d && d < M)) continue;
      if (!((M - d) * 1000000 < th * M)) continue;
      if (d >= target) continue;
      const int32_t u = W.slot_to_orig[s];
      const auto& ou = lout[u];
      // logical 2-hop out-neighbours q not in N+(u) + {u}, min combined weight
      std::vector<std::pair<int32_t, uint32_t>> two;
      for (const auto& ex : ou)
        for (const auto& eq : lout[ex.first]) {
          const int32_t q = eq.first;
          if (q == u) continue;
          if (std::binary_search(ou.begin(), ou.end(), std::make_pair(q, 0u),
                                 [](const std::pair<int32_t, uint32_t>& x, const std::pair<int32_t, uint32_t>& y) {
                                   return x.first < y.first;
                                 }))
            continue;
          two.push_back({q, combine_w(ex.second, eq.second, wrule)});
        }
      std::sort(two.begin(), two.end());   // by q, then weight: the first of each q is its minimum
      std::vector<std::pair<uint32_t, int32_t>> cand;
      for (size_t i = 0; i < two.size(); i++)
        if (i == 0 || two[i].first != two[i - 1].first) cand.push_back({two[i].second, two[i].first});
      std::sort(cand.begin(), cand.end());
      const int64_t take = std::min<int64_t>(target - d, (int64_t)cand.size());
      for (int64_t j = 0; j < take; j++) adds[s].push_back({W.owner[cand[j].second], cand[j].first, ADD_DEGNORM});
    }
  }
  pt("padding candidates");
  }
  added = 0;
#pragma omp parallel for schedule(dynamic, 4096) reduction(+ : added)
  for (int64_t s = 0; s < ns; s++) {
    added += (int64_t)adds[s].size();
    for (auto& e : adds[s]) W.rows[s].push_back(e);
  }
  par_free(adds);
  par_free(lout);
  sched = order;
  pt("padding applied + freed");
}

}  // namespace

void transform_host(const HostCSR& g, const gx_knobs& k, SlotGraph& out, Ctx* dev) {
  auto t0 = std::chrono::steady_clock::now();
  // GX_TRANSFORM_TRACE=1: per-phase host times on stderr
  const bool trace = getenv("GX_TRANSFORM_TRACE") != nullptr;
  auto tp = t0;
  auto phase = [&](const char* name) {
    if (!trace) return;
    auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "transform %-12s %8.1f ms\n", name, std::chrono::duration<double, std::milli>(now - tp).count());
    tp = now;
  };
  Work W;
  if (k.coalesce) coalesce(g, k.chunk_k, ppm(k.replicate_threshold), k.added_weight_rule, W, dev);
  else identity(g, W);
  phase(k.coalesce ? "coalesce" : "identity");
  SmemOut sm;
  if (k.smem) {
    Logical L;
    build_logical(W, L, dev);
    phase("logical+tri");
    const int64_t th = ppm(k.cc_threshold);
    const int64_t budget = k.added_edge_budget >= 0 ? k.added_edge_budget : g.m / 100;
    cc_edges(L, th, budget, k.added_weight_rule, k.sibling_undirected != 0, sm);
    phase("cc_edges");
    subgraphs(L, th, k.smem_max_nodes, k.smem_iters, sm);
    phase("subgraphs");
    for (auto& e : sm.added)
      W.rows[W.owner[std::get<0>(e)]].push_back({W.owner[std::get<1>(e)], std::get<2>(e), ADD_SMEM});
    phase("smem free");
  }
  std::vector<int32_t> sched;
  int64_t added_dn = 0;
  if (k.degree_norm)
    degnorm(W, ppm(k.degsim_threshold), ppm(k.degree_target), k.coalesce != 0, k.added_weight_rule, sched, added_dn,
            dev);
  phase("degnorm");

  // assemble the slot CSR, rows sorted by destination slot (R11)
  out = SlotGraph();
  out.n = W.n;
  out.n_slots = W.n_slots;
  out.rp.assign(W.n_slots + 1, 0);
  for (int64_t s = 0; s < W.n_slots; s++) out.rp[s + 1] = out.rp[s] + (int64_t)W.rows[s].size();
  out.m_slots = out.rp[W.n_slots];
  out.col.resize(out.m_slots);
  out.w.resize(out.m_slots);
  out.added.resize(out.m_slots);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t s = 0; s < W.n_slots; s++) {
    auto& r = W.rows[s];
    std::sort(r.begin(), r.end(), [](const Edge& a, const Edge& b) { return a.dst < b.dst; });
    int64_t o = out.rp[s];
    for (const Edge& e : r) {
      out.col[o] = e.dst;
      out.w[o] = e.w;
      out.added[o] = e.added;
      o++;
    }
  }
  out.slot_to_orig = W.slot_to_orig;
  out.kind = W.kind;
  out.owner_slot = W.owner;
  out.sched = sched;
  out.tile_ptr.assign(1, 0);
  for (auto& t : sm.tiles) {
    out.tile_centre.push_back(std::get<0>(t));
    for (int32_t v : std::get<1>(t)) out.tile_members.push_back(v);
    out.tile_ptr.push_back((int64_t)out.tile_members.size());
    out.tile_iters.push_back(std::get<2>(t));
  }
  phase("assemble");
  gx_transform_info& I = out.info;
  std::memset(&I, 0, sizeof(I));
  I.n_slots = W.n_slots;
  I.m_slots = out.m_slots;
  I.n_holes = W.n_holes;
  I.n_replicas = W.n_repl;
  I.holes_filled = W.n_repl;
  I.edges_added_coalesce = W.added_coal;
  I.edges_added_smem = (int64_t)sm.added.size();
  I.edges_added_degnorm = added_dn;
  I.n_subgraphs = (int64_t)sm.tiles.size();
  I.subgraph_vertices = (int64_t)out.tile_members.size();
  // extra space (Table 5 analogue): added slots and edges relative to n + m
  I.extra_space_pct = 100.0 * (double)((W.n_slots - W.n) + (out.m_slots - g.m)) / (double)std::max<int64_t>(1, g.n + g.m);
  I.transform_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

}  // namespace gx

namespace gx {

// The same three transforms with the slot graph resident in HBM (SURVEY.md
// §8(f) N1, dtransform.cu): relabel, replica candidates and rows, G_L and its
// undirected view, triangles, degree buckets, the warp schedule, padding and
// the final CSR rebuild run on the device; the host keeps the sequential
// decisions -- the cursor numbering (Alg 2 l.10-20), the choice of each
// level's h best replica candidates (Alg 2 l.24-27, R13/R14), the §3
// budgeted insertion and subgraph packing -- and the per-slot metadata
// (slot -> vertex, slot kind, vertex -> owner slot).  Output equals
// transform_host's bit for bit.
void transform_device(const HostCSR& g, const gx_knobs& k, SlotGraph& out, Ctx* dev, DevCSR din) {
  auto t0 = std::chrono::steady_clock::now();
  const bool trace = getenv("GX_TRANSFORM_TRACE") != nullptr;
  auto tp = t0;
  auto phase = [&](const char* name) {
    if (!trace) return;
    auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "transform %-18s %8.1f ms\n", name, std::chrono::duration<double, std::milli>(now - tp).count());
    tp = now;
  };
  const int64_t n = g.n;
  int64_t ns = n, n_holes = 0, n_repl = 0, added_coal = 0;
  std::vector<int32_t> s2o, owner;
  std::vector<uint8_t> kind;
  DEdges E;
  if (k.coalesce) {
    const int kk = k.chunk_k;
    std::vector<std::pair<int64_t, int64_t>> ranges;
    renumber(g, kk, owner, ns, ranges, dev);
    s2o.assign(ns, -1);
    kind.assign(ns, HOLE);
    for (int64_t u = 0; u < n; u++) {
      s2o[owner[u]] = (int32_t)u;
      kind[owner[u]] = OWNER;
    }
    phase("slot maps");
    dt_from_csr(dev, g, owner.data(), E, din.rp, din.col, din.w);
    phase("relabel (GPU)");
    dt_sort(dev, E, ns);
    phase("sort (GPU)");
    // chunks of levels >= 1 whose previous level has holes (Alg 2 l.21-23)
    const int64_t nchunks = (ns + kk - 1) / kk;
    std::vector<int32_t> nonhole(std::max<int64_t>(nchunks, 1), 0), chunk_lv(std::max<int64_t>(nchunks, 1), -1);
    for (int64_t s = 0; s < ns; s++)
      if (kind[s] != HOLE) nonhole[s / kk]++;
    const size_t nlv = ranges.size();
    std::vector<int64_t> lv_holes(nlv, 0);
    for (size_t li = 1; li < nlv; li++) {
      lv_holes[li] = std::max<int64_t>(0, ranges[li].first - ranges[li - 1].second);
      if (lv_holes[li] <= 0) continue;
      for (int64_t C = ranges[li].first / kk; C <= (ranges[li].second - 1) / kk; C++) chunk_lv[C] = (int32_t)li;
    }
    std::vector<DtCand> cands;
    dt_replica_candidates(dev, E, kk, chunk_lv, nonhole, ppm(k.replicate_threshold), cands);
    // per level, the h holes go to the candidates in (count desc, slot, chunk) order
    std::vector<std::vector<std::tuple<int64_t, int32_t, int64_t>>> per(nlv);
    for (const DtCand& c : cands) per[c.lv].push_back({-(int64_t)c.cnt, c.s, (int64_t)c.C});
    std::vector<DtAsg> asg;
    for (size_t li = 1; li < nlv; li++) {
      const int64_t h0 = ranges[li - 1].second, h1 = ranges[li].first;
      if (h1 <= h0 || per[li].empty()) continue;
      auto& cl = per[li];
      const size_t h = (size_t)(h1 - h0);
      if (cl.size() > h) {
        std::nth_element(cl.begin(), cl.begin() + h, cl.end());
        cl.resize(h);
      }
      std::sort(cl.begin(), cl.end());
      int64_t hole = h0;
      for (auto& c : cl) asg.push_back({std::get<1>(c), (int32_t)std::get<2>(c), hole++});
    }
    phase("replica candidates (GPU)");
    added_coal = dt_replicate(dev, E, ns, kk, asg, kind, k.added_weight_rule);
    for (const DtAsg& a : asg) {
      kind[a.hole] = REPLICA;
      s2o[a.hole] = s2o[a.s];
    }
    int64_t holes_left = 0;
    for (int64_t s = 0; s < ns; s++) holes_left += kind[s] == HOLE;
    n_repl = (int64_t)asg.size();
    n_holes = holes_left + n_repl;
    phase("replica rows (GPU)");
  } else {
    s2o.resize(n);
    owner.resize(n);
    std::iota(s2o.begin(), s2o.end(), 0);
    std::iota(owner.begin(), owner.end(), 0);
    kind.assign(n, OWNER);
    dt_from_csr(dev, g, nullptr, E, din.rp, din.col, din.w);
    phase("edges (GPU)");
  }
  DBuf ds2o;
  ds2o.alloc(dev, sizeof(int32_t) * std::max<int64_t>(ns, 1));
  if (ns) CUDA_OK(cudaMemcpyAsync(ds2o.p, s2o.data(), sizeof(int32_t) * ns, cudaMemcpyHostToDevice, dev->stream));
  SmemOut sm;
  if (k.smem) {
    // G_L, U and the triangle counts on the device; the greedy insertion
    // (P@31015-31268, R22-R26) and the packing (R27, R28) on the host
    Logical L;
    L.n = n;
    DBuf lp, ld, lw, lkey, np, nc, dT;
    dt_logical(dev, E, ds2o, n, lp, ld, lw, &lkey);
    const int64_t ml = E.m;
    const int64_t mu = dt_undirected(dev, n, lkey, ml, np, nc);
    lkey.reset();
    dT.alloc(dev, sizeof(int64_t) * std::max<int64_t>(n, 1));
    gpu_triangles_dev(dev, n, np.as<int64_t>(), nc.as<int32_t>(), mu, dT.as<unsigned long long>());
    phase("logical+U+tri (GPU)");
    // the flat bases straight into the Logical (no per-vertex containers)
    DBuf pairs;
    dt_pairs(dev, ld, lw, ml, pairs);
    ld.reset();
    lw.reset();
    cudaStream_t st = dev->stream;
    L.op.resize(n + 1);
    L.np.resize(n + 1);
    L.oe.resize(ml);
    L.ne.resize(mu);
    L.T.assign(n, 0);
    static_assert(sizeof(OutE) == 8, "OutE is {int32 dst, uint32 w}");
    CUDA_OK(cudaMemcpyAsync(L.op.data(), lp.p, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost, st));
    CUDA_OK(cudaMemcpyAsync(L.np.data(), np.p, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost, st));
    if (ml) CUDA_OK(cudaMemcpyAsync(L.oe.data(), pairs.p, sizeof(OutE) * ml, cudaMemcpyDeviceToHost, st));
    if (mu) CUDA_OK(cudaMemcpyAsync(L.ne.data(), nc.p, sizeof(int32_t) * mu, cudaMemcpyDeviceToHost, st));
    if (n) CUDA_OK(cudaMemcpyAsync(L.T.data(), dT.p, sizeof(int64_t) * n, cudaMemcpyDeviceToHost, st));
    CUDA_OK(cudaStreamSynchronize(st));
    lp.reset(); pairs.reset(); np.reset(); nc.reset(); dT.reset();
    L.init_overlays();
    phase("logical to host");
    const int64_t th = ppm(k.cc_threshold);
    const int64_t budget = k.added_edge_budget >= 0 ? k.added_edge_budget : g.m / 100;
    cc_edges(L, th, budget, k.added_weight_rule, k.sibling_undirected != 0, sm);
    phase("cc_edges");
    subgraphs(L, th, k.smem_max_nodes, k.smem_iters, sm);
    phase("subgraphs");
    std::vector<uint64_t> ak, av;
    ak.reserve(sm.added.size());
    av.reserve(sm.added.size());
    for (auto& e : sm.added) {
      ak.push_back(((uint64_t)(uint32_t)owner[std::get<0>(e)] << 32) | (uint32_t)owner[std::get<1>(e)]);
      av.push_back((uint64_t)std::get<2>(e) | ((uint64_t)ADD_SMEM << 32));
    }
    dt_append(dev, E, ak, av);
    phase("smem append");
  }
  std::vector<int32_t> sched;
  int64_t added_dn = 0;
  if (k.degree_norm) {
    dt_degnorm(dev, E, ns, n, kind, ds2o, owner, ppm(k.degsim_threshold), ppm(k.degree_target), k.coalesce != 0,
               k.added_weight_rule, sched, added_dn);
    phase("degnorm (GPU)");
  }
  out = SlotGraph();
  out.n = n;
  out.n_slots = ns;
  dt_export(dev, E, ns, out);
  out.slot_to_orig = std::move(s2o);
  out.kind = std::move(kind);
  out.owner_slot = std::move(owner);
  out.sched = std::move(sched);
  out.tile_ptr.assign(1, 0);
  for (auto& t : sm.tiles) {
    out.tile_centre.push_back(std::get<0>(t));
    for (int32_t v : std::get<1>(t)) out.tile_members.push_back(v);
    out.tile_ptr.push_back((int64_t)out.tile_members.size());
    out.tile_iters.push_back(std::get<2>(t));
  }
  phase("assemble (GPU)");
  gx_transform_info& I = out.info;
  std::memset(&I, 0, sizeof(I));
  I.n_slots = ns;
  I.m_slots = out.m_slots;
  I.n_holes = n_holes;
  I.n_replicas = n_repl;
  I.holes_filled = n_repl;
  I.edges_added_coalesce = added_coal;
  I.edges_added_smem = (int64_t)sm.added.size();
  I.edges_added_degnorm = added_dn;
  I.n_subgraphs = (int64_t)sm.tiles.size();
  I.subgraph_vertices = (int64_t)out.tile_members.size();
  I.extra_space_pct = 100.0 * (double)((ns - n) + (out.m_slots - g.m)) / (double)std::max<int64_t>(1, g.n + g.m);
  I.transform_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

}  // namespace gx
