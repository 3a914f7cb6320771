"""GPU parity of the transformed-graph sweeps with the oracle (SURVEY.md
§8(a) A2-A11): every Graffix knob, both sweep mappings (LB and the paper's
thread-per-vertex TPV), replica merges (mean / min) and the §3 local pass.

* SSSP: bit-exact with Dijkstra on G_L (the oracle's definition on the
  transformed graph), which Theorem E1 makes equal to Dijkstra on G.
* PageRank: L1 <= 1e-6 against the oracle's PageRank of G_L (Theorem E3).
"""
import numpy as np
import pytest

import graphgen
from golden_io import load
from gpu_util import ctx, upload
from oracle import algos as A
from oracle import transform as T
from oracle.graph import from_raw, graph_to_edgelist, sssp_source

pytestmark = pytest.mark.gpu

GRAPHS = {
    "rmat12": lambda: graphgen.rmat(12),
    "road48": lambda: graphgen.road(48),
    "uniform": lambda: graphgen.uniform(3000, 30000),
    "fig1_4": lambda: load("fig1_4.txt")[0],
}
KNOBS = {
    "coal": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.4),
    "coal_k4": T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.2),
    "smem": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=200),
    "degnorm": T.Knobs(degree_norm=True, degsim_threshold=0.5),
    "all": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.3,
                   degree_norm=True, degsim_threshold=0.5),
}


def knobs_c(kn, merge_op=0):
    import paper_conf_icpp_0001n20_b200 as gx
    d = {f: getattr(kn, f) for f in kn.__dataclass_fields__}
    d["merge_op"] = merge_op
    return gx.Knobs(**d)


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
@pytest.mark.parametrize("mapping", ["auto", "lb", "tpv", "vns", "lb_unpacked", "lb_dense"])
def test_sssp_transformed_bit_exact(gname, kname, mapping, monkeypatch):
    if mapping == "lb_unpacked":   # the {dst, w} stream C5 takes (26 id + 7 weight bits > 32)
        monkeypatch.setenv("GX_SSSP_NO_PACK", "1")
        mapping = "lb"
    if mapping == "lb_dense":      # every refill as the blocked dense relaxation (+ merge, no local pass)
        monkeypatch.setenv("GX_SSSP_DENSE", "1e-9")
        mapping = "lb"
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = KNOBS[kname]
    tg = T.transform(g, kn)
    s = sssp_source(g)
    want = A.sssp_dijkstra(tg.logical(), s)
    assert np.array_equal(want, A.sssp_dijkstra(graph_to_edgelist(g), s))     # E1
    G = upload(raw)
    info = G.transform(knobs_c(kn))
    assert info["n_replicas"] == tg.info["n_replicas"]
    r = G.run("sssp", source=-1, mapping=mapping)
    assert r["converged"] == 1
    got = G.download("dist")
    assert np.array_equal(got, want), f"{int(np.sum(got != want))} mismatches"


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
@pytest.mark.parametrize("mapping", ["lb", "tpv", "pb"])
def test_pagerank_transformed_l1(gname, kname, mapping):
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = KNOBS[kname]
    tg = T.transform(g, kn)
    want, _ = A.pagerank(tg.logical(), tol=1e-14)
    G = upload(raw)
    G.transform(knobs_c(kn))
    G.run("pagerank", tol=1e-11, max_iters=5000, mapping=mapping)
    got = G.download("rank")
    assert np.abs(got - want).sum() <= 1e-6


@pytest.mark.parametrize("gname", ["road48", "rmat12"])
def test_merge_min_sssp(gname):
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.0)
    G = upload(raw)
    G.transform(knobs_c(kn, merge_op=1))
    G.run("sssp")
    assert np.array_equal(G.download("dist"), A.sssp_dijkstra(graph_to_edgelist(g), sssp_source(g)))


def test_device_transform_export_matches_oracle():
    raw = graphgen.rmat(11)
    kn = KNOBS["all"]
    G = upload(raw)
    G.transform(knobs_c(kn))
    ex = G.export()
    tg = T.transform(from_raw(raw), kn)
    rp, col, w, ad = tg.csr()
    assert ex["n_slots"] == tg.n_slots
    assert np.array_equal(ex["row_ptr"], rp) and np.array_equal(ex["col"], col)
    assert np.array_equal(ex["w"].astype(np.int64), w) and np.array_equal(ex["slot_kind"], tg.slot_kind)


def test_inaccuracy_reporting():
    """Inaccuracy per knob (P@40990): SSSP exact at convergence (E1), PR not."""
    from oracle.metrics import inaccuracy
    raw = graphgen.rmat(12)
    G = upload(raw)
    G.run("sssp")
    d0 = G.download("dist")
    G.run("pagerank", tol=1e-12)
    x0 = G.download("rank")
    G.transform(knobs_c(KNOBS["all"]))
    G.run("sssp")
    G.run("pagerank", tol=1e-12)
    assert inaccuracy(G.download("dist"), d0)["inacc_pct"] == 0.0
    assert inaccuracy(G.download("rank"), x0)["inacc_pct"] > 0.0


@pytest.mark.parametrize("gname", ["road48", "rmat12"])
def test_pagerank_aware_merge_same_fixed_point(gname):
    """Algorithm-aware merge for PR (owner broadcast, R54) reaches the same G_L
    fixed point as the paper's mean merge (Theorem E3)."""
    raw = GRAPHS[gname]()
    kn = T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.0)
    want, _ = A.pagerank(T.transform(from_raw(raw), kn).logical(), tol=1e-14)
    G = upload(raw)
    G.transform(knobs_c(kn, merge_op=1))
    r = G.run("pagerank", tol=1e-11, max_iters=5000, mapping="lb")
    assert np.abs(G.download("rank") - want).sum() <= 1e-6


# ---------------------------------------------------------------- PR schedule + merge cadence (N2)
@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", ["coal", "smem", "all"])
@pytest.mark.parametrize("schedule", ["jacobi", "async"])
def test_pagerank_schedules_same_fixed_point(gname, kname, schedule):
    """Jacobi (two contrib buffers) and the asynchronous in-place schedule
    reach the same G_L PageRank (Theorem E3: any schedule)."""
    raw = GRAPHS[gname]()
    kn = KNOBS[kname]
    want, _ = A.pagerank(T.transform(from_raw(raw), kn).logical(), tol=1e-14)
    G = upload(raw)
    G.transform(knobs_c(kn))
    G.run("pagerank", tol=1e-11, max_iters=5000, mapping="lb", pr_schedule=schedule)
    assert np.abs(G.download("rank") - want).sum() <= 1e-6


@pytest.mark.parametrize("gname", ["road48", "rmat12", "fig1_4"])
@pytest.mark.parametrize("c", [2, 3, 0])
@pytest.mark.parametrize("mapping", ["lb", "tpv"])
def test_sssp_merge_cadence(gname, c, mapping):
    """c > 1 ends at the merged fixed point (= Dijkstra, E1); c = 0 ("merge at
    the end", P@28188) is bit-exact with the oracle's end-only loop."""
    from oracle import slotsim as S
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.0)
    tg = T.transform(g, kn)
    s = sssp_source(g)
    want = A.sssp_dijkstra(graph_to_edgelist(g), s) if c else S.sssp_slots(tg, s, merge_every=0, local_pass=False)[0]
    G = upload(raw)
    G.transform(knobs_c(kn))
    G.run("sssp", mapping=mapping, merge_every=c)
    got = G.download("dist")
    assert np.array_equal(got, want), f"{int(np.sum(got != want))} mismatches"


@pytest.mark.parametrize("gname", ["road48", "rmat12"])
@pytest.mark.parametrize("c", [2, 0])
@pytest.mark.parametrize("schedule", ["jacobi", "async", "async_pb"])
def test_pagerank_merge_cadence(gname, c, schedule):
    from oracle import slotsim as S
    raw = GRAPHS[gname]()
    kn = T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.0)
    tg = T.transform(from_raw(raw), kn)
    want = A.pagerank(tg.logical(), tol=1e-14)[0] if c else S.pagerank_slots(tg, tol=1e-14, merge_every=0)[0]
    G = upload(raw)
    G.transform(knobs_c(kn))
    mapping = "pb" if schedule == "async_pb" else "lb"
    G.run("pagerank", tol=1e-12, max_iters=20000, mapping=mapping, pr_schedule=schedule.split("_")[0],
          merge_every=c)
    assert np.abs(G.download("rank") - want).sum() <= 1e-6


# ---------------------------------------------------------------- N3 added-edge variants
N3 = {
    "coal_wmax": T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.2, added_weight="max"),
    "smem_und_wmean": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=300, sibling_undirected=True,
                              added_weight="mean"),
    "degnorm_wmax": T.Knobs(degree_norm=True, degsim_threshold=0.5, added_weight="max"),
    "all_und_wmax": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.3,
                            sibling_undirected=True, degree_norm=True, degsim_threshold=0.5, added_weight="max"),
}


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(N3))
@pytest.mark.parametrize("mapping", ["lb", "tpv"])
def test_n3_sssp_pagerank_on_GL(gname, kname, mapping):
    """Alternative weights / undirected siblings: the GPU still reaches the
    G_L definitions exactly (SSSP bit-exact with Dijkstra(G_L), PR within 1e-6),
    and SSSP may now be shorter than on G (never longer): non-zero inaccuracy."""
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = N3[kname]
    L = T.transform(g, kn).logical()
    s = sssp_source(g)
    want = A.sssp_dijkstra(L, s)
    exact = A.sssp_dijkstra(graph_to_edgelist(g), s)
    fin = exact != 0xFFFFFFFF
    assert np.all(want[fin] <= exact[fin])
    G = upload(raw)
    G.transform(knobs_c(kn))
    G.run("sssp", mapping=mapping)
    got = G.download("dist")
    assert np.array_equal(got, want), f"{int(np.sum(got != want))} mismatches"
    xw, _ = A.pagerank(L, tol=1e-14)
    G.run("pagerank", tol=1e-11, max_iters=5000, mapping=mapping)
    assert np.abs(G.download("rank") - xw).sum() <= 1e-6


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("variant", ["warp", "cta"])
@pytest.mark.parametrize("mapping", ["lb", "pb"])
def test_pagerank_local_pass_variants(gname, variant, mapping, monkeypatch):
    """The §3 PageRank local pass, one warp per tile (default, k_pr_local_warp)
    and one CTA per tile (GX_PR_LOCAL_CTA=1, k_pr_local): same fixed point
    (Theorem E3), within L1 1e-6 of the oracle's PageRank of G_L."""
    if variant == "cta":
        monkeypatch.setenv("GX_PR_LOCAL_CTA", "1")
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=-1)
    want, _ = A.pagerank(T.transform(g, kn).logical(), tol=1e-14)
    G = upload(raw)
    G.transform(knobs_c(kn))
    G.run("pagerank", mapping=mapping, tol=1e-11, max_iters=5000)
    assert np.abs(G.download("rank") - want).sum() <= 1e-6
