"""Seeded synthetic input graphs shared by the oracle and the CUDA path.

This module holds none of the Graffix method's arithmetic: it only emits a
raw directed CSR (duplicates and self-loops kept; each row ordered by
(destination, edge index)), which each side canonicalises on its own
(reading R2).  Recipes:

* ``rmat(scale)``   -- R-MAT, edge factor 16, (a,b,c,d) = (.45,.15,.15,.25)
  (GTgraph defaults; the paper's generator, PAPER.md P@35965), ids permuted.
* ``uniform(n, m)`` -- uniform random (src, dst) pairs ("random26").
* ``road(side)``    -- road-like lattice: spanning tree + 15% of the other
  lattice edges + 10% diagonals, symmetric, natural ids ("USA-road").
* weights: uniform integers 1..100 per edge index.

Seeds follow SURVEY.md §8(d): graph 20200817, weights 20200818.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "libgraphgen.so")

GRAPH_SEED = 20200817
WEIGHT_SEED = 20200818
BC_SEED = 20200819


def build(force: bool = False) -> str:
    """Compile gen.c into libgraphgen.so (gcc, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i64, u64, u32, i32 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        _lib.gg_rmat_edges.argtypes = [i32, i64, u64, u64, u32, u32, u32, i32, P, P, P]
        _lib.gg_uniform_edges.argtypes = [i64, i64, u64, u64, P, P, P]
        _lib.gg_road_edges.argtypes = [i64, u64, u64, P, P, P]
        _lib.gg_road_edges.restype = i64
        _lib.gg_build_csr.argtypes = [i64, i64, P, P, P, P, P, P]
    return _lib


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


@dataclass
class RawGraph:
    """Raw directed CSR as generated (before canonicalisation)."""
    n: int
    row_ptr: np.ndarray  # int64 [n+1]
    col: np.ndarray      # int32 [m]
    w: np.ndarray        # uint32 [m]
    name: str = ""

    @property
    def m(self) -> int:
        return int(self.col.shape[0])


def edges_to_csr(n: int, src: np.ndarray, dst: np.ndarray, w: np.ndarray, name: str = "") -> RawGraph:
    m = int(src.shape[0])
    assert m < 2**31, "edge index must fit 31 bits"
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    w = np.ascontiguousarray(w, dtype=np.uint32)
    row_ptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(m, dtype=np.int32)
    ow = np.empty(m, dtype=np.uint32)
    _L().gg_build_csr(n, m, _p(src), _p(dst), _p(w), _p(row_ptr), _p(col), _p(ow))
    return RawGraph(n, row_ptr, col, ow, name)


def rmat(scale: int, edge_factor: int = 16, seed: int = GRAPH_SEED, wseed: int = WEIGHT_SEED,
         abcd=(0.45, 0.15, 0.15, 0.25), permute: bool = True) -> RawGraph:
    n = 1 << scale
    m = edge_factor * n
    a, b, c, _ = abcd
    t = lambda x: min(int(round(x * 2**32)), 2**32 - 1)
    src = np.empty(m, np.int32); dst = np.empty(m, np.int32); w = np.empty(m, np.uint32)
    _L().gg_rmat_edges(scale, m, seed, wseed, t(a), t(a + b), t(a + b + c), int(permute), _p(src), _p(dst), _p(w))
    return edges_to_csr(n, src, dst, w, f"rmat{scale}")


def uniform(n: int, m: int, seed: int = GRAPH_SEED, wseed: int = WEIGHT_SEED) -> RawGraph:
    src = np.empty(m, np.int32); dst = np.empty(m, np.int32); w = np.empty(m, np.uint32)
    _L().gg_uniform_edges(n, m, seed, wseed, _p(src), _p(dst), _p(w))
    return edges_to_csr(n, src, dst, w, f"uniform{n}x{m}")


def road(side: int, seed: int = GRAPH_SEED, wseed: int = WEIGHT_SEED) -> RawGraph:
    L = _L()
    m = int(L.gg_road_edges(side, seed, wseed, None, None, None))
    src = np.empty(m, np.int32); dst = np.empty(m, np.int32); w = np.empty(m, np.uint32)
    L.gg_road_edges(side, seed, wseed, _p(src), _p(dst), _p(w))
    return edges_to_csr(side * side, src, dst, w, f"road{side}")


def from_edge_list(n: int, edges, name: str = "") -> RawGraph:
    """Tiny hand-written graphs: ``edges`` = [(u, v, w), ...] in row order.

    Unlike the generators, the given per-row order is preserved exactly
    (the §2 renumbering depends on adjacency order)."""
    rows = [[] for _ in range(n)]
    for e in edges:
        u, v = int(e[0]), int(e[1])
        ww = int(e[2]) if len(e) > 2 else 1
        rows[u].append((v, ww))
    row_ptr = np.zeros(n + 1, np.int64)
    for u in range(n):
        row_ptr[u + 1] = row_ptr[u] + len(rows[u])
    col = np.array([v for r in rows for v, _ in r], dtype=np.int32)
    w = np.array([ww for r in rows for _, ww in r], dtype=np.uint32)
    return RawGraph(n, row_ptr, col, w, name)


def bc_sources(n: int, k: int, seed: int = BC_SEED) -> np.ndarray:
    """K distinct seeded BC sources."""
    rng = np.random.default_rng(seed)
    k = min(k, n)
    return np.sort(rng.choice(n, size=k, replace=False)).astype(np.int64)
