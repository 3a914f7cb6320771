"""Pins for the oracle's algorithm definitions (CPU only).

Each oracle function is checked against something other than itself:
scipy / networkx routines, brute force on tiny graphs, closed forms and
invariants -- chosen so a dropped term, wrong sign/index or transposed
operand fails at least one test.
"""
import itertools

import networkx as nx
import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.csgraph as csg
from hypothesis import given, settings, strategies as st

import graphgen
from oracle import algos as A
from oracle import metrics as M
from oracle.graph import INF32, EdgeList, from_raw, graph_to_edgelist, sssp_source


def rand_el(seed, n, p, wmax=100):
    rng = np.random.default_rng(seed)
    s, d, w = [], [], []
    for u in range(n):
        for v in range(n):
            if u != v and rng.random() < p:
                s.append(u); d.append(v); w.append(int(rng.integers(1, wmax + 1)))
    return EdgeList(n, np.array(s, np.int64), np.array(d, np.int64), np.array(w, np.int64))


def nxg(el, directed=True):
    G = nx.DiGraph() if directed else nx.Graph()
    G.add_nodes_from(range(el.n))
    for u, v, w in zip(el.src.tolist(), el.dst.tolist(), el.w.tolist()):
        G.add_edge(u, v, weight=w)
    return G


# ---------------------------------------------------------------- SSSP
@settings(max_examples=60, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(1, 25), p=st.floats(0.0, 0.5))
def test_sssp_vs_bellman_ford_and_scipy(seed, n, p):
    el = rand_el(seed, n, p)
    s = seed % n
    dist = A.sssp_dijkstra(el, s)
    # Bellman-Ford brute force
    bf = [float("inf")] * n
    bf[s] = 0
    for _ in range(n):
        for u, v, w in zip(el.src, el.dst, el.w):
            if bf[u] + w < bf[v]:
                bf[v] = bf[u] + w
    want = np.array([INF32 if x == float("inf") else x for x in bf], dtype=np.uint64)
    assert np.array_equal(dist.astype(np.uint64), want)
    if el.src.size:
        mat = sp.csr_matrix((el.w.astype(float), (el.src, el.dst)), shape=(n, n))
        sc = csg.dijkstra(mat, directed=True, indices=s)
        sc = np.where(np.isinf(sc), INF32, sc).astype(np.uint64)
        assert np.array_equal(dist.astype(np.uint64), sc)


def test_sssp_grid_manhattan_closed_form():
    side = 17
    s, d = [], []
    for r in range(side):
        for c in range(side):
            v = r * side + c
            for dr, dc in ((0, 1), (1, 0), (0, -1), (-1, 0)):
                rr, cc = r + dr, c + dc
                if 0 <= rr < side and 0 <= cc < side:
                    s.append(v); d.append(rr * side + cc)
    el = EdgeList(side * side, np.array(s), np.array(d), np.ones(len(s), np.int64))
    src = 5 * side + 3
    dist = A.sssp_dijkstra(el, src)
    for r in range(side):
        for c in range(side):
            assert dist[r * side + c] == abs(r - 5) + abs(c - 3)


def test_sssp_certificate_accepts_and_rejects():
    g = from_raw(graphgen.rmat(10))
    s = sssp_source(g)
    dist = A.sssp_dijkstra(graph_to_edgelist(g), s)
    assert M.sssp_certificate(g, s, dist)["ok"]
    bad = dist.copy()
    v = int(np.nonzero((bad != INF32) & (np.arange(g.n) != s))[0][0])
    bad[v] += 1
    assert not M.sssp_certificate(g, s, bad)["ok"]
    bad = dist.copy(); bad[v] -= 1
    assert not M.sssp_certificate(g, s, bad)["ok"]


def test_sssp_source_rule():
    g = from_raw(graphgen.from_edge_list(4, [(1, 0, 1), (1, 2, 1), (3, 0, 1), (3, 1, 1)]))
    assert sssp_source(g) == 1   # max out-degree 2, ties to the lowest id


# ---------------------------------------------------------------- PageRank
def dense_pr(el, d=0.85):
    n = el.n
    dout = np.bincount(el.src, minlength=n).astype(float)
    Mx = np.zeros((n, n))
    for u, v in zip(el.src, el.dst):
        Mx[v, u] += 1.0 / dout[u]
    for u in range(n):
        if dout[u] == 0:
            Mx[:, u] += 1.0 / n
    return np.linalg.solve(np.eye(n) - d * Mx, np.full(n, (1 - d) / n))


@settings(max_examples=40, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(1, 30), p=st.floats(0.0, 0.4))
def test_pagerank_vs_dense_solve(seed, n, p):
    el = rand_el(seed, n, p)
    x, _ = A.pagerank(el)
    assert np.abs(x - dense_pr(el)).sum() < 1e-11
    assert abs(x.sum() - 1.0) < 1e-12


def test_pagerank_vs_networkx_and_closed_forms():
    el = graph_to_edgelist(from_raw(graphgen.rmat(9)))
    x, _ = A.pagerank(el)
    ref = nx.pagerank(nxg(el), alpha=0.85, weight=None, tol=1e-13, max_iter=10000)
    assert np.abs(x - np.array([ref[v] for v in range(el.n)])).sum() < 1e-9
    n = 7
    cyc = EdgeList(n, np.arange(n), (np.arange(n) + 1) % n, np.ones(n, np.int64))
    assert np.allclose(A.pagerank(cyc)[0], 1.0 / n, atol=1e-14)
    s, d = zip(*[(a, b) for a in range(n) for b in range(n) if a != b])
    comp = EdgeList(n, np.array(s), np.array(d), np.ones(len(s), np.int64))
    assert np.allclose(A.pagerank(comp)[0], 1.0 / n, atol=1e-14)
    # one dangling sink fed by all others: closed form by symmetry
    s = np.arange(1, n); d = np.zeros(n - 1, np.int64)
    x, _ = A.pagerank(EdgeList(n, s, d, np.ones(n - 1, np.int64)))
    assert np.abs(x - dense_pr(EdgeList(n, s, d, np.ones(n - 1, np.int64)))).sum() < 1e-12
    assert x[0] > x[1] and np.allclose(x[1:], x[1])


def test_pagerank_residual_certificate():
    el = graph_to_edgelist(from_raw(graphgen.rmat(10)))
    x, _ = A.pagerank(el)
    r = M.pagerank_residual(el.src, el.dst, el.n, x)
    assert r["bound"] < 1e-11 and abs(r["mass"] - 1) < 1e-12
    r2 = M.pagerank_residual(el.src, el.dst, el.n, np.full(el.n, 1.0 / el.n))
    assert r2["bound"] > 1e-3


# ---------------------------------------------------------------- SCC
@settings(max_examples=60, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(1, 10), p=st.floats(0.0, 0.5))
def test_scc_vs_closure_brute_force(seed, n, p):
    el = rand_el(seed, n, p)
    R = np.eye(n, dtype=bool)
    for u, v in zip(el.src, el.dst):
        R[u, v] = True
    for kk in range(n):
        R = R | (R[:, [kk]] & R[[kk], :])
    want = np.array([min(v for v in range(n) if R[u, v] and R[v, u]) for u in range(n)])
    lab = A.scc_tarjan(el)
    assert np.array_equal(lab, want)
    assert np.array_equal(lab[lab], lab)


def test_scc_vs_networkx():
    el = graph_to_edgelist(from_raw(graphgen.rmat(10)))
    lab = A.scc_tarjan(el)
    want = np.empty(el.n, np.int64)
    for comp in nx.strongly_connected_components(nxg(el)):
        mn = min(comp)
        for v in comp:
            want[v] = mn
    assert np.array_equal(lab, want)


# ---------------------------------------------------------------- MST
@settings(max_examples=40, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(1, 7), p=st.floats(0.0, 0.6))
def test_mst_vs_exhaustive(seed, n, p):
    el = rand_el(seed, n, p, wmax=9)
    best = {}
    for u, v, w in zip(el.src.tolist(), el.dst.tolist(), el.w.tolist()):
        key = (min(u, v), max(u, v))
        best[key] = min(w, best.get(key, 10**9))
    edges = list(best.items())
    G = nx.Graph(); G.add_nodes_from(range(n)); G.add_edges_from(best)
    ncomp = nx.number_connected_components(G)
    r = n - ncomp
    opt = None
    for sub in itertools.combinations(edges, r):
        H = nx.Graph(); H.add_nodes_from(range(n)); H.add_edges_from(e for e, _ in sub)
        if nx.is_forest(H) and nx.number_connected_components(H) == ncomp:
            tot = sum(w for _, w in sub)
            opt = tot if opt is None else min(opt, tot)
    assert A.mst_kruskal(el) == (opt or 0)


def test_mst_vs_networkx():
    el = graph_to_edgelist(from_raw(graphgen.rmat(10)))
    G = nx.Graph()
    G.add_nodes_from(range(el.n))
    for u, v, w in zip(el.src.tolist(), el.dst.tolist(), el.w.tolist()):
        if not G.has_edge(u, v) or G[u][v]["weight"] > w:
            G.add_edge(u, v, weight=w)
    F = nx.minimum_spanning_tree(G, algorithm="prim")
    assert A.mst_kruskal(el) == int(F.size(weight="weight"))


# ---------------------------------------------------------------- BC
def bc_brute(el, sources):
    """Enumerate all shortest paths by BFS-DAG path counting per (s, t)."""
    n = el.n
    adj = [[] for _ in range(n)]
    for u, v in zip(el.src.tolist(), el.dst.tolist()):
        adj[u].append(v)

    def paths(s):
        dist = {s: 0}; order = [s]
        for u in order:
            for v in adj[u]:
                if v not in dist:
                    dist[v] = dist[u] + 1; order.append(v)
        # enumerate all shortest paths explicitly
        allp = {s: [[s]]}
        for u in order[1:]:
            allp[u] = [p + [u] for x in range(n) if x in dist and dist[x] == dist[u] - 1
                       and u in adj[x] for p in allp[x]]
        return allp
    bc = np.zeros(n)
    for s in sources:
        allp = paths(int(s))
        for t, ps in allp.items():
            if t == s:
                continue
            for p in ps:
                for v in p[1:-1]:
                    bc[v] += 1.0 / len(ps)
    return bc


@settings(max_examples=40, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(1, 9), p=st.floats(0.0, 0.6))
def test_bc_vs_path_enumeration(seed, n, p):
    el = rand_el(seed, n, p)
    srcs = list(range(0, n, 2))
    assert np.allclose(A.bc_brandes(el, srcs), bc_brute(el, srcs), atol=1e-12)


def test_bc_vs_networkx_all_sources_and_invariant():
    el = graph_to_edgelist(from_raw(graphgen.rmat(8)))
    bc = A.bc_brandes(el, range(el.n))
    ref = nx.betweenness_centrality(nxg(el), normalized=False)
    assert np.allclose(bc, [ref[v] for v in range(el.n)], rtol=1e-10, atol=1e-9)
    # sum_v bc[v] = sum_s sum_t (hops(s,t) - 1) over reachable pairs
    srcs = graphgen.bc_sources(el.n, 8)
    bc = A.bc_brandes(el, srcs)
    G = nxg(el)
    tot = sum(h - 1 for s in srcs for t, h in nx.single_source_shortest_path_length(G, int(s)).items()
              if t != s)
    assert abs(bc.sum() - tot) < 1e-6 * max(1, tot)


# ---------------------------------------------------------------- metrics
def test_inaccuracy_definition():
    e = np.array([1.0, 2.0, 3.0]); a = np.array([1.0, 2.5, 2.0])
    r = M.inaccuracy(a, e)
    assert abs(r["inacc_pct"] - 100 * 1.5 / 6) < 1e-12 and abs(r["mae"] - 0.5) < 1e-12
    assert M.inaccuracy(e, e)["inacc_pct"] == 0.0
    d = np.array([0, 5, INF32], np.uint32); d2 = np.array([0, 6, 7], np.uint32)
    r = M.inaccuracy(d2, d)
    assert r["inf_mismatch"] == 1 and abs(r["inacc_pct"] - 20.0) < 1e-12
    assert M.inaccuracy(11, 10, "scalar")["inacc_pct"] == pytest.approx(10.0)


def test_canonicalize_sorted_matches_canonicalize():
    from oracle.graph import canonicalize_sorted
    for G in [graphgen.rmat(11), graphgen.uniform(2000, 40000), graphgen.road(40)]:
        a = from_raw(G)
        b = canonicalize_sorted(G.n, G.row_ptr, G.col, G.w)
        assert np.array_equal(a.row_ptr, b.row_ptr) and np.array_equal(a.col, b.col)
        assert np.array_equal(a.w, b.w)
