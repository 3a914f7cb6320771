"""Theorems E1-E4, pinned on random transformed graphs.

The slot execution (oracle.slotsim: Jacobi sweep + local pass + mean merge,
the paper's loop) must reach exactly the G_L definitions in oracle.algos,
and under the sum-weight rule the SSSP/SCC/MST results on G_L equal those on
the original graph G (so their inaccuracy is 0 at convergence, reading R42).
"""
import numpy as np
from hypothesis import given, settings, strategies as st

import graphgen
from oracle import algos as A
from oracle import slotsim as S
from oracle import transform as T
from oracle.graph import from_raw, graph_to_edgelist


def rand_graph(seed, n, p):
    rng = np.random.default_rng(seed)
    edges = [(u, v, int(rng.integers(1, 101))) for u in range(n) for v in range(n)
             if u != v and rng.random() < p]
    return from_raw(graphgen.from_edge_list(n, edges))


KNOBS = [
    T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.3),
    T.Knobs(coalesce=True, chunk_k=2, replicate_threshold=0.0),
    T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=20, smem_max_nodes=10),
    T.Knobs(degree_norm=True, degsim_threshold=0.6),
    T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.2, smem=True, cc_threshold=0.2,
            added_edge_budget=10, degree_norm=True, degsim_threshold=0.6),
]


@settings(max_examples=50, deadline=None)
@given(seed=st.integers(0, 10**6), n=st.integers(2, 24), p=st.floats(0.05, 0.35),
       ki=st.integers(0, len(KNOBS) - 1))
def test_E1_E3_slot_execution_reaches_GL(seed, n, p, ki):
    g = rand_graph(seed, n, p)
    tg = T.transform(g, KNOBS[ki])
    L = tg.logical()
    src = seed % n
    d_slot, _ = S.sssp_slots(tg, src)
    d_L = A.sssp_dijkstra(L, src)
    d_G = A.sssp_dijkstra(graph_to_edgelist(g), src)
    assert np.array_equal(d_slot, d_L)          # slot execution = Dijkstra(G_L)
    assert np.array_equal(d_L, d_G)             # E1: = Dijkstra(G)
    x_slot, _ = S.pagerank_slots(tg)
    x_L, _ = A.pagerank(L)
    assert np.abs(x_slot - x_L).sum() < 1e-9    # E3
    # E2 / E4
    assert np.array_equal(A.scc_tarjan(L), A.scc_tarjan(graph_to_edgelist(g)))
    assert A.mst_kruskal(L) == A.mst_kruskal(graph_to_edgelist(g))


def test_E1_on_rmat_with_all_knobs():
    g = from_raw(graphgen.rmat(8))
    kn = T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.3, smem=True,
                 cc_threshold=0.3, degree_norm=True, degsim_threshold=0.5)
    tg = T.transform(g, kn)
    s = int(np.argmax(g.outdeg()))
    d_slot, _ = S.sssp_slots(tg, s)
    assert np.array_equal(d_slot, A.sssp_dijkstra(graph_to_edgelist(g), s))
