"""Oracle: the three Graffix graph transforms, step by step.

Test infrastructure only (see oracle/__init__.py).  Readings R# are those of
SURVEY.md §8(c) c3, restated in DESIGN.md; thresholds are compared in
integer parts-per-million (ppm = floor(x * 1e6 + 0.5)).

* §2 coalescing, Alg 2 (P@16373-18419; text P@19014-27600):
    renumber()   -- BFS-forest levels (l.2-6) + RenumberVertex (l.10-20)
    replicate()  -- ReplicateVertex (l.21-35): copies into holes, moved
                    edges, 2-hop edges; confluence groups (§2.4 P@27655).
* §3 memory latency (P@29857-32416): local clustering coefficient on the
    undirected view, CC-raising sibling edges under a global budget, and
    disjoint shared-memory subgraphs {c} + N(c) processed t ~ 2*diam times.
* §4 thread divergence (P@33145-35029): degree buckets, warps in bucket
    order, 2-hop padding to ceil(0.85 * warp max) when degreeSim < theta.

Composition §2 -> §3 -> §4 (reading R34).  Exact mode = identity.
Parity status:
  renumber/replicate: pinned to the Fig 1-4 printed example (tests/golden)
    and to the isomorphism / 2-hop-path invariants;
  degree padding: pinned to the Fig 6 example + invariants;
  cc_edges (case 1 / case 2 selection) and subgraph packing: pinned to six
    hand-derived fixtures (tests/golden/sec3_*.txt, derivations in each file,
    P@31015 common-neighbour preference, P@31268 fewest internal edges) that
    kill every single-decision mutant of tools/mutate_sec3.py, plus the
    invariants (budget, 2-path + sum weight, disjointness).  Fig 5 itself
    cannot be recovered; the selection rules R22-R28 are readings.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from math import floor

import numpy as np

from .graph import EdgeList, Graph

OWNER, REPLICA, HOLE = 0, 1, 2
ADD_NONE, ADD_COALESCE, ADD_SMEM, ADD_DEGNORM = 0, 1, 2, 3


def ppm(x: float) -> int:
    return int(floor(float(x) * 1e6 + 0.5))


@dataclass
class Knobs:
    """Mirrors gx_knobs (include/graffix.h); all techniques off = exact mode."""
    coalesce: bool = False
    chunk_k: int = 16                    # k = 16 (P@25752)
    replicate_threshold: float = 0.6     # connectedness theta (P@25752; 0.4 road)
    smem: bool = False
    cc_threshold: float = 0.5
    added_edge_budget: int = -1          # <0 => 1% of m (reading R26)
    smem_iters: int = 0                  # 0 => 2 * diameter (P@32282)
    smem_max_nodes: int = 64             # S_max (reading R27)
    degree_norm: bool = False
    degsim_threshold: float = 0.3        # best near 0.3 (P@55324)
    degree_target: float = 0.85          # 85% of warp max (P@55220)
    added_weight: str = "sum"            # N3: weight rule of every added edge (combine())
    sibling_undirected: bool = False     # N3: §3 sibling edges on the undirected CC view


WEIGHT_RULES = ("sum", "max", "mean")


def combine(w1: int, w2: int, rule: str = "sum") -> int:
    """Weight of an added edge u->q that stands for the 2-hop path u->v->q
    with hop weights w1, w2.  P@34493 sets it to the sum ("sum", reading R17,
    the default: the edge is never shorter than the path it replaces) and
    P@34692 allows "an alternative method to set up the edge-weights"
    (SURVEY N3): "max" = the heavier hop, "mean" = floor((w1 + w2) / 2),
    at least 1.  Any rule but "sum" can shorten distances (inexact SSSP)."""
    if rule == "sum":
        return w1 + w2
    if rule == "max":
        return max(w1, w2)
    if rule == "mean":
        return max(1, (w1 + w2) // 2)
    raise ValueError(rule)


@dataclass
class TransformedGraph:
    n: int                               # original vertices
    n_slots: int
    slot_to_orig: np.ndarray             # int64 [n_slots], -1 for holes
    slot_kind: np.ndarray                # uint8 [n_slots] OWNER/REPLICA/HOLE
    owner_slot: np.ndarray               # int64 [n] (new id of each vertex)
    rows: list                           # per slot: list of [dst_slot, w, added]
    sched: np.ndarray                    # lane -> slot (§4); identity if off
    tiles: list = field(default_factory=list)   # (centre, members(sorted orig ids), t)
    info: dict = field(default_factory=dict)
    levels: list = field(default_factory=list)  # §2: per level (start, end) slot range
    sources: list = field(default_factory=list) # §2: BFS-forest sources (orig ids)

    # -- views ---------------------------------------------------------------
    def logical(self) -> EdgeList:
        """G_L: every slot edge with its source mapped to the owner vertex."""
        s, d, w, a = [], [], [], []
        for slot, row in enumerate(self.rows):
            u = int(self.slot_to_orig[slot])
            for (q, ww, ad) in row:
                s.append(u); d.append(int(self.slot_to_orig[q])); w.append(ww); a.append(ad)
        return EdgeList(self.n, np.asarray(s, np.int64), np.asarray(d, np.int64),
                        np.asarray(w, np.int64), np.asarray(a, np.int64))

    def csr(self):
        """Slot CSR, rows sorted by destination slot (reading R11)."""
        rp = np.zeros(self.n_slots + 1, np.int64)
        col, w, ad = [], [], []
        for s, row in enumerate(self.rows):
            r = sorted(row)
            rp[s + 1] = rp[s] + len(r)
            for q, ww, a in r:
                col.append(q); w.append(ww); ad.append(a)
        return rp, np.asarray(col, np.int64), np.asarray(w, np.int64), np.asarray(ad, np.int64)

    def groups(self):
        """Confluence groups: owner slot -> [owner slot] + replica slots."""
        g = {}
        for s in range(self.n_slots):
            if self.slot_kind[s] == REPLICA:
                o = int(self.owner_slot[self.slot_to_orig[s]])
                g.setdefault(o, [o]).append(s)
        return g

    def divisor(self) -> np.ndarray:
        """D[slot] = total logical out-degree of the slot's vertex (§8(c) c1 §2.6)."""
        deg = np.zeros(self.n, np.int64)
        for s, row in enumerate(self.rows):
            if self.slot_kind[s] != HOLE:
                deg[self.slot_to_orig[s]] += len(row)
        D = np.zeros(self.n_slots, np.int64)
        for s in range(self.n_slots):
            if self.slot_kind[s] != HOLE:
                D[s] = deg[self.slot_to_orig[s]]
        return D


# ----------------------------------------------------------------------------
# identity (exact mode)
# ----------------------------------------------------------------------------
def identity(g: Graph) -> TransformedGraph:
    adj = g.adjacency_lists()
    rows = [[[v, w, ADD_NONE] for (v, w) in adj[u]] for u in range(g.n)]
    ids = np.arange(g.n, dtype=np.int64)
    return TransformedGraph(g.n, g.n, ids.copy(), np.zeros(g.n, np.uint8), ids.copy(), rows,
                            ids.copy())


# ----------------------------------------------------------------------------
# §2 step 1: levels + renumbering (Alg 2 l.1-20)
# ----------------------------------------------------------------------------
def bfs_forest_levels(g: Graph):
    """Alg 2 l.2-6 (P@16484) with readings R3-R5.

    Sources: vertices in (out-degree desc, id asc) order (R3); a vertex not
    yet reached starts a new BFS over out-edges (reachability marking).
    level[v] = multi-source BFS distance from the source set (R4: later BFS
    runs lower levels, P@20759).  Returns (sources in selection order, level).
    """
    n = g.n
    adj = [[v for v, _ in r] for r in g.adjacency_lists()]
    deg = [len(a) for a in adj]
    order = sorted(range(n), key=lambda v: (-deg[v], v))
    visited = [False] * n
    sources = []
    for s in order:
        if visited[s]:
            continue
        sources.append(s)
        visited[s] = True
        stack = [s]
        while stack:
            u = stack.pop()
            for v in adj[u]:
                if not visited[v]:
                    visited[v] = True
                    stack.append(v)
    level = [-1] * n
    frontier = list(sources)
    for s in sources:
        level[s] = 0
    lv = 0
    while frontier:
        nxt = []
        for u in frontier:
            for v in adj[u]:
                if level[v] < 0:
                    level[v] = lv + 1
                    nxt.append(v)
        frontier = nxt
        lv += 1
    return sources, level


def renumber(g: Graph, k: int):
    """RenumberVertex (Alg 2 l.10-20, P@16766; text P@21573-22978).

    L0 gets ids 0..|L0|-1 in source-selection order (R5).  For each level i:
    gId = ceil(gId/k)*k (l.14; the skipped slots are holes); the parents
    L_i in ascending new id (R8) take turns, round robin, each numbering the
    next not-yet-numbered level-(i+1) vertex of its adjacency list in CSR
    order (the cursor reading R6/R7: "all first neighbours, then second ..."
    P@21936); rounds stop when one assigns nothing.  After the last level the
    slot count is padded to a multiple of k (R9).
    Returns (new_of_old, n_slots, levels[(start, end)], sources).
    """
    n = g.n
    sources, level = bfs_forest_levels(g)
    adj = [[v for v, _ in r] for r in g.adjacency_lists()]
    new = [-1] * n
    for i, v in enumerate(sources):
        new[v] = i
    gid = len(sources)
    ranges = [(0, gid)]
    cur = list(sources)
    i = 0
    while True:
        start = -(-gid // k) * k
        parents = sorted(cur, key=lambda v: new[v])
        cursor = [0] * len(parents)
        nxt = []
        gid2 = start
        while True:
            assigned = False
            for pi, p in enumerate(parents):
                row = adj[p]
                c = cursor[pi]
                while c < len(row) and not (level[row[c]] == i + 1 and new[row[c]] == -1):
                    c += 1
                if c < len(row):
                    new[row[c]] = gid2
                    gid2 += 1
                    nxt.append(row[c])
                    c += 1
                    assigned = True
                cursor[pi] = c
            if not assigned:
                break
        if not nxt:
            break
        ranges.append((start, gid2))
        gid = gid2
        cur = nxt
        i += 1
    n_slots = -(-gid // k) * k if n > 0 else 0
    assert all(x >= 0 for x in new)
    return np.asarray(new, np.int64), n_slots, ranges, sources


def coalesce(g: Graph, k: int, theta_ppm: int, rule: str = "sum") -> TransformedGraph:
    """§2: renumber into an isomorph, then ReplicateVertex (Alg 2 l.21-35).

    Replication (P@17298-18419, P@23832-27600, readings R10-R18):
      * holes of level i-1 are the slots [end_{i-1}, start_i) (R10);
      * for every level i >= 1 whose level i-1 has h > 0 holes, every chunk C
        (chunk(s) = s // k, l.21) of level i and every non-hole vertex n:
        count = #edges n->p with chunk(p) = C; (n, C) is a candidate iff
        count * 1e6 >= theta_ppm * nonhole(C)  (l.28 ">=", R13;
        connectedness P@24839);
      * candidates sorted (count desc, n's new id asc, C asc) (R14); the first
        h take level i-1's holes in ascending slot order; a vertex may be
        replicated more than once (R15);
      * per assignment (n, C, hole): every edge n->p with chunk(p) = C moves to
        the hole's row (l.32-34); the hole gets n->q for every non-hole q in C
        with q not in N+(n) + {n} reachable as n->v->q, weight
        min_v combine(w(n,v), w(v,q)) (l.35; R16, R17; sum by default),
        using n's pre-move edges;
      * replicas have no in-edges (R18).
    """
    new, n_slots, ranges, sources = renumber(g, k)
    n = g.n
    adj = g.adjacency_lists()
    slot_to_orig = np.full(n_slots, -1, np.int64)
    slot_to_orig[new] = np.arange(n)
    kind = np.full(n_slots, HOLE, np.uint8)
    kind[new] = OWNER
    # renumbered adjacency (slot ids), in original CSR order
    radj = {}
    for u in range(n):
        radj[int(new[u])] = [(int(new[v]), w) for (v, w) in adj[u]]
    rows = [[] for _ in range(n_slots)]
    for s, r in radj.items():
        rows[s] = [[q, w, ADD_NONE] for (q, w) in r]

    def nonhole(C):
        return sum(1 for s in range(C * k, min(C * k + k, n_slots)) if kind[s] != HOLE)

    n_repl = 0
    added = 0
    assignments = []
    for i in range(1, len(ranges)):
        holes = list(range(ranges[i - 1][1], ranges[i][0]))
        if not holes:
            continue
        c_lo = ranges[i][0] // k
        c_hi = (ranges[i][1] - 1) // k
        cnt = {}
        for s, r in radj.items():
            for (q, _) in r:
                C = q // k
                if c_lo <= C <= c_hi:
                    cnt[(s, C)] = cnt.get((s, C), 0) + 1
        cands = []
        for (s, C), c in cnt.items():
            if c * 1_000_000 >= theta_ppm * nonhole(C):
                cands.append((-c, s, C))
        cands.sort()
        for (negc, s, C), h in zip(cands, holes):
            assignments.append((s, C, h))
    for (s, C, h) in assignments:
        orig_row = radj[s]
        nplus = {q for (q, _) in orig_row}
        moved = [[q, w, ADD_NONE] for (q, w) in orig_row if q // k == C]
        rows[s] = [e for e in rows[s] if e[0] // k != C]
        best = {}
        for (v, wv) in orig_row:
            for (q, wq) in radj[v]:
                if q // k == C and q not in nplus and q != s and kind[q] != HOLE:
                    wc = combine(wv, wq, rule)
                    if q not in best or wc < best[q]:
                        best[q] = wc
        rows[h] = moved + [[q, w, ADD_COALESCE] for q, w in sorted(best.items())]
        kind[h] = REPLICA
        slot_to_orig[h] = slot_to_orig[s]
        n_repl += 1
        added += len(best)
    n_holes = int(np.sum(kind == HOLE)) + n_repl
    tg = TransformedGraph(n, n_slots, slot_to_orig, kind, new, rows,
                          np.arange(n_slots, dtype=np.int64), levels=ranges, sources=sources)
    tg.info.update(n_holes=n_holes, n_replicas=n_repl, holes_filled=n_repl,
                   edges_added_coalesce=added)
    return tg


# ----------------------------------------------------------------------------
# §3: clustering coefficient, sibling edges, subgraphs
# ----------------------------------------------------------------------------
class _Logical:
    """Mutable logical graph (original ids) with its undirected view U."""

    def __init__(self, tg: TransformedGraph):
        n = tg.n
        self.out = [dict() for _ in range(n)]
        self.inn = [dict() for _ in range(n)]
        for slot, row in enumerate(tg.rows):
            if tg.slot_kind[slot] == HOLE:
                continue
            u = int(tg.slot_to_orig[slot])
            for (q, w, _) in row:
                v = int(tg.slot_to_orig[q])
                self.out[u][v] = w
                self.inn[v][u] = w
        self.N = [set(self.out[u]) | set(self.inn[u]) for u in range(n)]
        self.T = [self._tri(u) for u in range(n)]

    def _tri(self, c):
        Nc = self.N[c]
        t = 0
        for a in Nc:
            t += len(self.N[a] & Nc)
        return t // 2

    def P(self, c):
        d = len(self.N[c])
        return d * (d - 1) // 2

    def high(self, c, th):
        # strict >, CC = 0 when d < 2 (reading R21)
        return self.T[c] * 1_000_000 > th * self.P(c)

    def eligible(self, c, a, b, undirected=False):
        """Sibling edge a->b for centre c: along a directed 2-path a->c->b
        (reading R23); with undirected=True (N3, the CC view P@29950) any
        two neighbours of c in U."""
        if undirected:
            return a in self.N[c] and b in self.N[c]
        return (c in self.out[a]) and (b in self.out[c])

    def wU(self, a, b):
        """Weight of the pair {a, b} in U: the lighter existing direction."""
        ws = [x for x in (self.out[a].get(b), self.out[b].get(a)) if x is not None]
        return min(ws)

    def link(self, a, b, w):
        """Insert a->b into G_L; keep N and triangle counts current."""
        newly_adj = b not in self.N[a]
        self.out[a][b] = w
        self.inn[b][a] = w
        if newly_adj:
            common = self.N[a] & self.N[b]
            for x in common:
                self.T[x] += 1
            self.T[a] += len(common)
            self.T[b] += len(common)
            self.N[a].add(b)
            self.N[b].add(a)


def cc_edges(tg: TransformedGraph, cc_ppm: int, budget: int, rule: str = "sum", undirected: bool = False):
    """§3 edge insertion (P@30608-32051), readings R21-R26.  Pinned by the
    hand-derived fixtures S1-S6 (tests/golden/sec3_*.txt): centre order
    (S1), pair order by common neighbours P@31015 (S2), stop at high (S2),
    case-2 sibling / partner by fewest internal edges P@31268 (S3), case 1
    before case 2 and case-2 centre order (S4), skip rule (S5), round-robin
    passes (S6); tools/mutate_sec3.py shows each decision is load-bearing.

    Case 1 (raise near-threshold centres, R22): non-high centres with d >= 2
    in (need asc, id asc) order, need = floor(theta_ppm * P / 1e6) + 1 - T
    from the state before §3; at each visit need / T / linkable pairs are
    recomputed; a centre with fewer linkable pairs than need is skipped;
    else pairs are linked in (|N(a) & N(b)| desc, a asc, b asc) order (order
    fixed at the visit) until the centre is high or the budget is spent.
    Case 2 (boost high centres, R24/R25): with the remaining budget,
    round-robin passes over the centres high after case 1 in (CC desc, id asc)
    order; per centre per pass one pair: the sibling a with the smallest
    internal degree |N(a) & N(c)| (ties: id) having a linkable partner, joined
    to its lowest-internal-degree linkable partner (ties: id).  Stops when
    the budget is 0 or a pass links nothing.
    Linking {a, b} inserts a->b if eligible then b->a if eligible (a < b),
    each costing 1 unit of budget, weight combine(w(x,c), w(c,y)) (sum rule
    R17 by default).  undirected=True (N3): every pair of U-neighbours of c
    is eligible in both directions, hop weights taken in U (wU).
    Returns the list of added (a, b, w)."""
    L = _Logical(tg)
    n = tg.n
    added = []
    rem = [budget]

    def linkable(c, a, b):
        return b not in L.N[a] and (L.eligible(c, a, b, undirected) or L.eligible(c, b, a, undirected))

    def do_link(c, a, b):
        for (x, y) in ((a, b), (b, a)):
            if rem[0] <= 0:
                return
            if L.eligible(c, x, y, undirected) and y not in L.out[x]:
                if undirected:
                    w = combine(L.wU(x, c), L.wU(c, y), rule)
                else:
                    w = combine(L.out[x][c], L.out[c][y], rule)
                L.link(x, y, w)
                added.append((x, y, w))
                rem[0] -= 1

    # case 1
    cands = []
    for c in range(n):
        d = len(L.N[c])
        if d >= 2 and not L.high(c, cc_ppm):
            need = (cc_ppm * L.P(c)) // 1_000_000 + 1 - L.T[c]
            cands.append((need, c))
    cands.sort()
    for _, c in cands:
        if rem[0] <= 0:
            break
        P = L.P(c)
        need = (cc_ppm * P) // 1_000_000 + 1 - L.T[c]
        if need <= 0:
            continue
        if P - L.T[c] < need:
            continue
        Nc = sorted(L.N[c])
        pairs = []
        for i, a in enumerate(Nc):
            for b in Nc[i + 1:]:
                if linkable(c, a, b):
                    pairs.append((-len(L.N[a] & L.N[b]), a, b))
        if len(pairs) < need:
            continue
        pairs.sort()
        for _, a, b in pairs:
            if rem[0] <= 0 or L.high(c, cc_ppm):
                break
            if linkable(c, a, b):
                do_link(c, a, b)
    # case 2
    if rem[0] > 0:
        highs = [c for c in range(n) if L.high(c, cc_ppm)]
        # CC desc by exact rational compare, id asc
        from functools import cmp_to_key

        def cmp(x, y):
            lhs = L.T[x] * L.P(y)
            rhs = L.T[y] * L.P(x)
            if lhs != rhs:
                return -1 if lhs > rhs else 1
            return -1 if x < y else (1 if x > y else 0)
        highs.sort(key=cmp_to_key(cmp))
        while rem[0] > 0:
            linked_any = False
            for c in highs:
                if rem[0] <= 0:
                    break
                Nc = L.N[c]
                intdeg = {a: len(L.N[a] & Nc) for a in Nc}
                sib = sorted(Nc, key=lambda a: (intdeg[a], a))
                done = False
                for a in sib:
                    partners = [b for b in Nc if b != a and linkable(c, a, b)]
                    if partners:
                        b = min(partners, key=lambda x: (intdeg[x], x))
                        x, y = (a, b) if a < b else (b, a)
                        do_link(c, x, y)
                        done = True
                        break
                linked_any |= done
            if not linked_any:
                break
    return added, L


def subgraphs(L: _Logical, n: int, cc_ppm: int, smax: int, smem_iters: int):
    """§3 shared-memory subgraphs (P@30023-30382, P@31631, P@32188-32416),
    readings R27/R28.  Pinned by the tiles of fixtures S1-S6 (centre order
    CC desc S1, d desc S2, id asc S1/S4; t = 2 x diameter: 2 for cliques,
    4 in S3/S4/S6).

    Centres: high vertices with 1 + d <= S_max, ordered (CC desc (exact
    rational), d desc, id asc); S(c) = {c} + N(c) is accepted iff disjoint from
    the subgraphs already accepted.  t = 2 * undirected diameter of U[S(c)]
    (clique -> 1, else 2), or smem_iters when > 0."""
    from functools import cmp_to_key
    cs = [c for c in range(n) if L.high(c, cc_ppm) and 1 + len(L.N[c]) <= smax]

    def cmp(x, y):
        lhs = L.T[x] * L.P(y)
        rhs = L.T[y] * L.P(x)
        if lhs != rhs:
            return -1 if lhs > rhs else 1
        dx, dy = len(L.N[x]), len(L.N[y])
        if dx != dy:
            return -1 if dx > dy else 1
        return -1 if x < y else (1 if x > y else 0)
    cs.sort(key=cmp_to_key(cmp))
    used = set()
    tiles = []
    for c in cs:
        S = {c} | L.N[c]
        if S & used:
            continue
        used |= S
        d = len(L.N[c])
        clique = L.T[c] == d * (d - 1) // 2
        t = smem_iters if smem_iters > 0 else 2 * (1 if clique else 2)
        tiles.append((c, sorted(S), t))
    return tiles


def apply_smem(tg: TransformedGraph, knobs: Knobs, m_orig: int):
    cc_ppm = ppm(knobs.cc_threshold)
    budget = knobs.added_edge_budget if knobs.added_edge_budget >= 0 else m_orig // 100
    added, L = cc_edges(tg, cc_ppm, budget, knobs.added_weight, knobs.sibling_undirected)
    for (a, b, w) in added:
        tg.rows[int(tg.owner_slot[a])].append([int(tg.owner_slot[b]), w, ADD_SMEM])
    tg.tiles = subgraphs(L, tg.n, cc_ppm, knobs.smem_max_nodes, knobs.smem_iters)
    tg.info["edges_added_smem"] = len(added)
    tg.info["n_subgraphs"] = len(tg.tiles)
    tg.info["subgraph_vertices"] = sum(len(t[1]) for t in tg.tiles)


# ----------------------------------------------------------------------------
# §4: degree buckets + warp-level padding
# ----------------------------------------------------------------------------
def bucket(d: int) -> int:
    """Reading R30: 0 for d = 0, else 1 + floor(log2 d)."""
    return int(d).bit_length()


def apply_degnorm(tg: TransformedGraph, knobs: Knobs, combined: bool):
    """§4 (P@33145-35029, P@54828-55273), readings R30-R34.

    Degrees are slot out-degrees after §2/§3 (R33).  Standalone: order =
    non-hole slots stable-sorted by bucket desc (R30); combined with §2:
    order = slot order (R34).  Warps = consecutive 32 entries (R31).  In each
    warp M = max d; an owner slot v with 0 < d < M and
    (M - d) * 1e6 < theta_ppm * M (degreeSim < theta, R32) whose d < target =
    ceil(f_ppm * M / 1e6) gets up to target - d edges v->q to logical 2-hop
    out-neighbours q not in N+(v) + {v} (non-hole), ordered by
    (min_x combine(w(v,x), w(x,q)), q asc); candidates come from the graph before any
    §4 addition.  Replica slots are not padded (reading)."""
    th = ppm(knobs.degsim_threshold)
    f = ppm(knobs.degree_target)
    deg = [len(r) for r in tg.rows]
    if combined:
        order = list(range(tg.n_slots))
    else:
        ns = [s for s in range(tg.n_slots) if tg.slot_kind[s] != HOLE]
        order = sorted(ns, key=lambda s: (-bucket(deg[s]), s))
    # pre-§4 logical out adjacency
    lout = [dict() for _ in range(tg.n)]
    for slot, row in enumerate(tg.rows):
        if tg.slot_kind[slot] == HOLE:
            continue
        u = int(tg.slot_to_orig[slot])
        for (q, w, _) in row:
            lout[u][int(tg.slot_to_orig[q])] = w
    adds = []
    for base in range(0, len(order), 32):
        lanes = order[base:base + 32]
        M = max(deg[s] for s in lanes)
        target = (f * M + 999_999) // 1_000_000
        for s in lanes:
            d = deg[s]
            if tg.slot_kind[s] != OWNER or not (0 < d < M):
                continue
            if not ((M - d) * 1_000_000 < th * M):
                continue
            if d >= target:
                continue
            u = int(tg.slot_to_orig[s])
            best = {}
            for x, wx in lout[u].items():
                for q, wq in lout[x].items():
                    if q == u or q in lout[u]:
                        continue
                    wc = combine(wx, wq, knobs.added_weight)
                    if q not in best or wc < best[q]:
                        best[q] = wc
            cand = sorted(best.items(), key=lambda kv: (kv[1], kv[0]))[:target - d]
            for q, w in cand:
                adds.append((s, int(tg.owner_slot[q]), w))
    for (s, qs, w) in adds:
        tg.rows[s].append([qs, w, ADD_DEGNORM])
    tg.sched = np.asarray(order, np.int64)
    tg.info["edges_added_degnorm"] = len(adds)


# ----------------------------------------------------------------------------
def transform(g: Graph, knobs: Knobs | None = None) -> TransformedGraph:
    """TransformGraph (Alg 2 l.1-9) extended with §3 and §4 (composition R34)."""
    knobs = knobs or Knobs()
    if knobs.coalesce:
        tg = coalesce(g, knobs.chunk_k, ppm(knobs.replicate_threshold), knobs.added_weight)
    else:
        tg = identity(g)
        tg.info.update(n_holes=0, n_replicas=0, holes_filled=0, edges_added_coalesce=0)
    tg.info.setdefault("edges_added_smem", 0)
    tg.info.setdefault("n_subgraphs", 0)
    tg.info.setdefault("subgraph_vertices", 0)
    if knobs.smem:
        apply_smem(tg, knobs, g.m)
    tg.info.setdefault("edges_added_degnorm", 0)
    if knobs.degree_norm:
        apply_degnorm(tg, knobs, combined=knobs.coalesce)
    tg.info["n_slots"] = tg.n_slots
    return tg
