"""Oracle: the plain definitions each algorithm computes.

Test infrastructure only (see oracle/__init__.py).  Every function takes a
logical graph as parallel (src, dst, w) arrays over original vertex ids; for
a transformed graph that is G_L (oracle.transform.TransformedGraph.logical()).
"""
from __future__ import annotations

import heapq
from collections import deque

import numpy as np

from .graph import INF32, EdgeList


def _csr(n, src, dst, w=None):
    order = np.lexsort((dst, src))
    rp = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rp, np.asarray(src, dtype=np.int64) + 1, 1)
    rp = np.cumsum(rp)
    d = np.asarray(dst, dtype=np.int64)[order]
    ww = None if w is None else np.asarray(w, dtype=np.int64)[order]
    return rp, d, ww


def sssp_dijkstra(g: EdgeList, source: int) -> np.ndarray:
    """O1: single-source shortest path distances, Dijkstra with a binary heap.

    The paper's SSSP (P@37923, attribute "distance" P@41178) with integer
    weights; unreachable = 2^32-1 (reading R36).  Pinned in tests against
    scipy.sparse.csgraph.dijkstra, Bellman-Ford brute force and the
    grid Manhattan closed form."""
    n = g.n
    rp, d, w = _csr(n, g.src, g.dst, g.w)
    rp = rp.tolist(); d = d.tolist(); w = w.tolist()
    dist = [None] * n
    dist_best = [float("inf")] * n
    dist_best[source] = 0
    heap = [(0, source)]
    while heap:
        du, u = heapq.heappop(heap)
        if dist[u] is not None:
            continue
        dist[u] = du
        for e in range(rp[u], rp[u + 1]):
            v = d[e]
            nd = du + w[e]
            if dist[v] is None and nd < dist_best[v]:
                dist_best[v] = nd
                heapq.heappush(heap, (nd, v))
    out = np.full(n, INF32, dtype=np.uint64)
    for v in range(n):
        if dist[v] is not None:
            out[v] = dist[v]
    return out.astype(np.uint32)


def pagerank(g: EdgeList, damping: float = 0.85, tol: float = 1e-13, max_iters: int = 100000):
    """O3: PageRank by fp64 power iteration (reading R35).

    x0 = 1/N;  x'_v = (1-d)/N + d * ( sum_{u->v} x_u / Dout(u)
                                       + sum_{Dout(u)=0} x_u / N ),
    stop when ||x' - x||_1 < tol.  Returns (x, iterations).  Pinned in tests
    against the dense solve of (I - d M) x = b, networkx.pagerank and the
    directed-cycle / complete-graph closed forms."""
    n = g.n
    src = np.asarray(g.src, dtype=np.int64)
    dst = np.asarray(g.dst, dtype=np.int64)
    dout = np.bincount(src, minlength=n).astype(np.float64)
    dangling = dout == 0
    x = np.full(n, 1.0 / n)
    for it in range(1, max_iters + 1):
        contrib = np.where(dangling, 0.0, x / np.where(dangling, 1.0, dout))
        y = np.bincount(dst, weights=contrib[src], minlength=n)
        xn = (1.0 - damping) / n + damping * (y + x[dangling].sum() / n)
        delta = np.abs(xn - x).sum()
        x = xn
        if delta < tol:
            return x, it
    return x, max_iters


def scc_tarjan(g: EdgeList) -> np.ndarray:
    """O2: strongly connected components (Tarjan, iterative).

    label[v] = the minimum original id in v's SCC (reading R38).  Pinned in
    tests against Kosaraju-by-closure brute force and networkx."""
    n = g.n
    rp, d, _ = _csr(n, g.src, g.dst)
    rp = rp.tolist(); d = d.tolist()
    index = [-1] * n; low = [0] * n; onstack = [False] * n
    stack = []; label = [-1] * n; counter = 0
    for root in range(n):
        if index[root] != -1:
            continue
        work = [(root, rp[root])]
        index[root] = low[root] = counter; counter += 1
        stack.append(root); onstack[root] = True
        while work:
            v, e = work[-1]
            if e < rp[v + 1]:
                work[-1] = (v, e + 1)
                u = d[e]
                if index[u] == -1:
                    index[u] = low[u] = counter; counter += 1
                    stack.append(u); onstack[u] = True
                    work.append((u, rp[u]))
                elif onstack[u]:
                    low[v] = min(low[v], index[u])
            else:
                work.pop()
                if work:
                    p = work[-1][0]
                    low[p] = min(low[p], low[v])
                if low[v] == index[v]:
                    comp = []
                    while True:
                        x = stack.pop(); onstack[x] = False; comp.append(x)
                        if x == v:
                            break
                    mn = min(comp)
                    for x in comp:
                        label[x] = mn
    return np.asarray(label, dtype=np.int64)


def mst_kruskal(g: EdgeList) -> int:
    """O4: total weight of the minimum spanning forest of the undirected view.

    {u,v} weighs min(w(u,v), w(v,u)) (reading R39); Kruskal with ties broken
    by (w, min(u,v), max(u,v)); union-find.  Pinned in tests against
    exhaustive enumeration (n <= 7), Prim and networkx."""
    n = g.n
    best = {}
    for u, v, w in zip(np.asarray(g.src).tolist(), np.asarray(g.dst).tolist(), np.asarray(g.w).tolist()):
        if u == v:
            continue
        a, b = (u, v) if u < v else (v, u)
        if (a, b) not in best or w < best[(a, b)]:
            best[(a, b)] = w
    parent = list(range(n))

    def find(x):
        while parent[x] != x:
            parent[x] = parent[parent[x]]
            x = parent[x]
        return x

    total = 0
    for (a, b), w in sorted(best.items(), key=lambda kv: (kv[1], kv[0][0], kv[0][1])):
        ra, rb = find(a), find(b)
        if ra != rb:
            parent[ra] = rb
            total += w
    return int(total)


def bc_brandes(g: EdgeList, sources) -> np.ndarray:
    """O5: betweenness centrality, Brandes (Alg 1, P@13282-14843).

    Unweighted, directed; sigma in fp64; for each source s: BFS forward pass
    building sigma and predecessor lists, backward pass
        delta_s(v) = sum_{w : v in pred_s(w)} sigma_sv / sigma_sw * (1 + delta_s(w))
    (Eq 1, P@12652) and bc[v] = sum_{s != v} delta_s(v) (Eq 2, P@13228), over
    the given source sample (reading R37).  Pinned in tests against
    networkx.betweenness_centrality_subset and path-enumeration brute force."""
    n = g.n
    rp, d, _ = _csr(n, g.src, g.dst)
    rp = rp.tolist(); d = d.tolist()
    bc = np.zeros(n, dtype=np.float64)
    for s in sources:
        s = int(s)
        sigma = [0.0] * n; dist = [-1] * n; pred = [[] for _ in range(n)]
        sigma[s] = 1.0; dist[s] = 0
        order = []; q = deque([s])
        while q:
            v = q.popleft(); order.append(v)
            for e in range(rp[v], rp[v + 1]):
                u = d[e]
                if dist[u] < 0:
                    dist[u] = dist[v] + 1; q.append(u)
                if dist[u] == dist[v] + 1:
                    sigma[u] += sigma[v]; pred[u].append(v)
        delta = [0.0] * n
        for wv in reversed(order):
            for v in pred[wv]:
                delta[v] += sigma[v] / sigma[wv] * (1.0 + delta[wv])
            if wv != s:
                bc[wv] += delta[wv]
    return bc
