"""Oracle: the paper's iteration on slots, for pinning Theorems E1 / E3.

Test infrastructure only (see oracle/__init__.py).  This is a plain
simulation of the execution model the GPU path follows -- a Jacobi sweep
over every slot edge ("main fixed-point loop repeatedly calling the primary
kernel", P@40883), the optional shared-memory local pass (P@32188-32416,
reading R29: after the sweep, before the merge), then confluence: the copies
of a vertex are set to the arithmetic mean of their values after every
iteration (§2.4, P@28309 / P@28609) with the mirror reading R19 (replicas
are not recomputed; integers take the floor of the exact mean; SSSP
excludes INF copies).  Tests use it to check that the slot execution reaches
exactly the G_L definitions in oracle.algos.
"""
from __future__ import annotations

import numpy as np

from .graph import INF32
from .transform import HOLE, TransformedGraph


def _merge_int(vals):
    fin = [v for v in vals if v != INF32]
    if not fin:
        return INF32
    return sum(fin) // len(fin)


def _merge_now(it: int, merge_every: int, sweep_fixed: bool) -> bool:
    """Merge cadence, P@28188: "The merging or the confluence may be done after
    a certain number of iterations or at the end of the overall computation"
    (Graffix's default: after every iteration).  merge_every = c: c == 1 every
    iteration; c > 1 after every c-th iteration (1-based) and after any
    iteration whose sweep changed nothing (so the run ends merged); c == 0 only
    "at the end": after the first iteration whose sweep changed nothing."""
    if merge_every == 1:
        return True
    if merge_every > 1 and it % merge_every == 0:
        return True
    return sweep_fixed


def sssp_slots(tg: TransformedGraph, source: int, max_iters: int = 100000,
               merge: str = "mean", local_pass: bool = True, merge_every: int = 1):
    """Returns (dist per original vertex, iterations).  With merge_every == 0
    the run ends right after its single final merge (values pushed by that
    merge are not relaxed further)."""
    groups = tg.groups()
    dist = [INF32] * tg.n_slots
    o = int(tg.owner_slot[source])
    for s in groups.get(o, [o]):
        dist[s] = 0
    it = 0
    while it < max_iters:
        it += 1
        new = list(dist)
        for s, row in enumerate(tg.rows):
            if dist[s] == INF32:
                continue
            for (q, w, _) in row:
                if dist[s] + w < new[q]:
                    new[q] = dist[s] + w
        if local_pass and tg.tiles:
            member_edges = {}
            for c, members, t in tg.tiles:
                ms = set(int(tg.owner_slot[v]) for v in members)
                for _ in range(t):
                    for s in ms:
                        if new[s] == INF32:
                            continue
                        for (q, w, _) in tg.rows[s]:
                            if q in ms and new[s] + w < new[q]:
                                new[q] = new[s] + w
        merged = bool(groups) and _merge_now(it, merge_every, new == dist)
        if merged:
            for own, copies in groups.items():
                mval = _merge_int([new[c] for c in copies]) if merge == "mean" else min(new[c] for c in copies)
                for c in copies:
                    new[c] = mval
        if merge_every == 0 and merged:
            dist = new
            break
        if new == dist and (merged or not groups):
            break
        dist = new
    return np.asarray([dist[int(tg.owner_slot[v])] for v in range(tg.n)], dtype=np.uint32), it


def pagerank_slots(tg: TransformedGraph, damping: float = 0.85, tol: float = 1e-13,
                   max_iters: int = 100000, merge_every: int = 1):
    """Mirror-replica PageRank on slots: each copy divides by D (the total
    logical out-degree); replicas carry the last merged value.  Returns
    (x per original vertex, iterations).  Merge cadence as in _merge_now, with
    "the sweep changed nothing" read as delta < tol."""
    N = tg.n
    groups = tg.groups()
    D = tg.divisor().astype(np.float64)
    x = np.zeros(tg.n_slots)
    live = tg.slot_kind != HOLE
    x[live] = 1.0 / N
    owners = np.asarray([int(tg.owner_slot[v]) for v in range(N)], dtype=np.int64)
    src, dst = [], []
    for s, row in enumerate(tg.rows):
        for (q, _, _) in row:
            src.append(s); dst.append(q)
    src = np.asarray(src, np.int64); dst = np.asarray(dst, np.int64)
    for it in range(1, max_iters + 1):
        contrib = np.where(D > 0, x / np.where(D > 0, D, 1.0), 0.0)
        y = np.bincount(dst, weights=contrib[src], minlength=tg.n_slots)
        dang = x[owners][D[owners] == 0].sum()
        xn = x.copy()
        xn[owners] = (1.0 - damping) / N + damping * (y[owners] + dang / N)
        sweep_fixed = np.abs(xn[owners] - x[owners]).sum() < tol
        merged = bool(groups) and _merge_now(it, merge_every, sweep_fixed)
        if merged:
            for own, copies in groups.items():
                xn[copies] = xn[copies].mean()
        delta = np.abs(xn[owners] - x[owners]).sum()
        x = xn
        if merge_every == 0 and merged:
            break
        if delta < tol and (merged or not groups):
            break
    return x[owners], it
