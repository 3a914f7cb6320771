"""Oracle: canonical graph and the logical graph G_L.

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

INF32 = 0xFFFFFFFF


@dataclass
class Graph:
    """A directed graph in CSR form: row u = col[row_ptr[u]:row_ptr[u+1]].

    CSR with offset / edges / edge-attribute arrays as in PAPER.md P@15127
    (§2.1, Fig 1).  The graph is directed (reading R1)."""
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    w: np.ndarray

    @property
    def m(self) -> int:
        return int(self.col.shape[0])

    def outdeg(self) -> np.ndarray:
        return np.diff(self.row_ptr).astype(np.int64)

    def row(self, u: int):
        a, b = int(self.row_ptr[u]), int(self.row_ptr[u + 1])
        return self.col[a:b], self.w[a:b]

    def edges(self):
        """(src, dst, w) arrays in CSR order."""
        src = np.repeat(np.arange(self.n, dtype=np.int64), self.outdeg())
        return src, self.col.astype(np.int64), self.w.astype(np.int64)

    def adjacency_lists(self):
        """Python lists [(v, w), ...] per row, in CSR order."""
        rp = self.row_ptr.tolist(); c = self.col.tolist(); w = self.w.tolist()
        return [list(zip(c[rp[u]:rp[u + 1]], w[rp[u]:rp[u + 1]])) for u in range(self.n)]


def canonicalize(n, row_ptr, col, w=None) -> Graph:
    """Canonical CSR (reading R2; the paper is silent).

    * self-loops are dropped;
    * a duplicate (u, v) is merged into its FIRST occurrence's position and
      keeps the minimum weight over the duplicates;
    * the surviving edges of each row keep the caller's order (the §2
      cursor walks adjacency in input order, P@21936 / App. A.1).
    ``w`` None means all weights 1.
    """
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    m = col.shape[0]
    w = np.ones(m, dtype=np.int64) if w is None else np.asarray(w, dtype=np.int64)
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(row_ptr))
    keep = src != col                                   # drop self-loops
    idx = np.nonzero(keep)[0]
    key = src[idx] * np.int64(n) + col[idx]
    order = np.lexsort((idx, key))                      # group duplicates, by position
    skey = key[order]
    first = np.ones(skey.shape[0], dtype=bool)
    first[1:] = skey[1:] != skey[:-1]
    starts = np.nonzero(first)[0]
    wmin = np.minimum.reduceat(w[idx][order], starts) if starts.size else np.zeros(0, np.int64)
    pos = idx[order][starts]                            # first occurrence positions
    o2 = np.argsort(pos, kind="stable")                 # restore input order
    pos = pos[o2]; wmin = wmin[o2]
    nsrc = src[pos]
    new_rp = np.zeros(n + 1, dtype=np.int64)
    np.add.at(new_rp, nsrc + 1, 1)
    new_rp = np.cumsum(new_rp)
    return Graph(n, new_rp, col[pos].astype(np.int64), wmin.astype(np.int64))


def from_raw(raw) -> Graph:
    """Canonicalise a graphgen.RawGraph."""
    return canonicalize(raw.n, raw.row_ptr, raw.col, raw.w)


def sssp_source(g: Graph) -> int:
    """Reading R36: the max-out-degree vertex, ties to the lowest id."""
    d = g.outdeg()
    return int(np.argmax(d)) if g.n else 0


@dataclass
class EdgeList:
    """A logical directed graph as parallel arrays (original vertex ids)."""
    n: int
    src: np.ndarray
    dst: np.ndarray
    w: np.ndarray
    added: np.ndarray = field(default=None)   # 0 original, >0 added by §2/§3/§4

    def to_graph(self) -> Graph:
        order = np.lexsort((self.dst, self.src))
        rp = np.zeros(self.n + 1, dtype=np.int64)
        np.add.at(rp, self.src + 1, 1)
        return Graph(self.n, np.cumsum(rp), self.dst[order].astype(np.int64),
                     self.w[order].astype(np.int64))


def graph_to_edgelist(g: Graph) -> EdgeList:
    s, d, w = g.edges()
    return EdgeList(g.n, s, d, w, np.zeros(s.shape[0], dtype=np.int64))


def canonicalize_sorted(n, row_ptr, col, w) -> Graph:
    """Same result as canonicalize() when every row is already ordered by
    destination (graphgen emits rows ordered by (destination, edge index), so
    duplicates are adjacent and the first occurrence is the first of its run).
    Vectorised for full-size (10^8-10^9 edge) checks; tests pin it to
    canonicalize() on generated graphs.  Raises if a row is not sorted."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col)
    w = np.asarray(w)
    m = col.shape[0]
    src = np.repeat(np.arange(n, dtype=np.int32), np.diff(row_ptr))
    same_row = np.zeros(m, dtype=bool)
    same_row[1:] = src[1:] == src[:-1]
    if np.any(same_row[1:] & (col[1:] < col[:-1])):
        raise ValueError("rows are not sorted by destination")
    dup = np.zeros(m, dtype=bool)
    dup[1:] = same_row[1:] & (col[1:] == col[:-1])
    run_start = np.nonzero(~dup)[0]
    wmin = np.minimum.reduceat(w, run_start) if m else w[:0]
    keep = run_start[src[run_start] != col[run_start]]
    wk = wmin[src[run_start] != col[run_start]]
    ksrc = src[keep]
    new_rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(ksrc, minlength=n), out=new_rp[1:])
    return Graph(n, new_rp, col[keep], wk)
