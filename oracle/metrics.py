"""Oracle: inaccuracy metric and O(m) certificates for full-size checks.

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np

from .graph import INF32, Graph


def inaccuracy(approx, exact, kind: str = "vector") -> dict:
    """Inaccuracy (P@40990-41294, reading R40).

    vector (SSSP distance, PR rank, BC value): over vertices finite in both
    runs, inacc% = 100 * sum|a - e| / sum|e|, plus the mean absolute error,
    the mean relative error and the count of INF/finite mismatches.
    scalar (SCC component count, MST weight): 100 * |a - e| / e."""
    if kind == "scalar":
        a, e = float(approx), float(exact)
        return {"inacc_pct": 100.0 * abs(a - e) / e if e else 0.0, "approx": a, "exact": e}
    a = np.asarray(approx); e = np.asarray(exact)
    if a.dtype == np.uint32 or e.dtype == np.uint32:
        fa = a != INF32; fe = e != INF32
        both = fa & fe
        mism = int(np.sum(fa != fe))
        a = a[both].astype(np.float64); e = e[both].astype(np.float64)
    else:
        mism = 0
        a = a.astype(np.float64); e = e.astype(np.float64)
    diff = np.abs(a - e)
    se = np.abs(e).sum()
    nz = np.abs(e) > 0
    return {
        "inacc_pct": float(100.0 * diff.sum() / se) if se > 0 else 0.0,
        "mae": float(diff.mean()) if diff.size else 0.0,
        "mean_rel": float(np.mean(diff[nz] / np.abs(e[nz]))) if nz.any() else 0.0,
        "inf_mismatch": mism,
    }


def sssp_certificate(g: Graph, source: int, dist: np.ndarray) -> dict:
    """O(m) SSSP certificate: dist[s] = 0; for every edge
    u->v with finite dist[u]: dist[v] <= dist[u] + w; every finite v != s has
    a tight in-edge (dist[v] = dist[u] + w); INF exactly on the unreachable
    set follows from the two.  Together these fix dist = the unique
    shortest-path distances (weights >= 1)."""
    dist = np.asarray(dist, dtype=np.int64)
    n = g.n
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(g.row_ptr))
    du = dist[src]
    fin = du != INF32
    cand = du[fin] + np.asarray(g.w, np.int64)[fin]
    dv = dist[np.asarray(g.col, np.int64)[fin]]
    violations = int(np.sum(dv > cand))
    tight = np.zeros(n, dtype=bool)
    tv = np.asarray(g.col, np.int64)[fin][dv == cand]
    tight[tv] = True
    need = (dist != INF32)
    need[source] = False
    untight = int(np.sum(need & ~tight))
    return {"source_zero": bool(dist[source] == 0), "violations": violations,
            "untight": untight,
            "ok": bool(dist[source] == 0 and violations == 0 and untight == 0)}


def pagerank_residual(src, dst, n: int, x, damping: float = 0.85) -> dict:
    """PR certificate: r = ||x - F(x)||_1 bounds ||x - x*||_1 <= r / (1 - d)."""
    src = np.asarray(src, np.int64); dst = np.asarray(dst, np.int64)
    x = np.asarray(x, np.float64)
    dout = np.bincount(src, minlength=n).astype(np.float64)
    dang = dout == 0
    contrib = np.where(dang, 0.0, x / np.where(dang, 1.0, dout))
    y = np.bincount(dst, weights=contrib[src], minlength=n)
    fx = (1.0 - damping) / n + damping * (y + x[dang].sum() / n)
    r = float(np.abs(x - fx).sum())
    return {"residual": r, "bound": r / (1.0 - damping), "mass": float(x.sum())}
