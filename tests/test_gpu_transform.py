"""GPU-resident preprocessing: with a device context the
§3 triangle counts (the clustering coefficients of P@29857 that drive the CC
edge insertion and the subgraph selection) and the §2 source order,
reachability forest and multi-source BFS levels (Alg 2 l.2-6) and the §4
padding candidates (2-hop out-neighbours ranked by (weight, id), P@33654) are
computed on the GPU (gtransform.cu), and with a device context the whole slot
graph is built in HBM (dtransform.cu: relabel, replica candidates and rows,
G_L / U, degree buckets and warp schedule, padding, the CSR rebuild); the host
keeps the cursor numbering and the greedy decisions.  The exported transformed
graph must be bit-identical to the oracle's and to the host-only library path
(no device), element by element -- the triangle counts feed integer decisions
only."""
import numpy as np
import pytest

import graphgen
from golden_io import load
from gpu_util import ctx, upload
from oracle import transform as T
from test_transform_parity import assert_same, oracle_export

pytestmark = pytest.mark.gpu

GRAPHS = {
    "rmat12": lambda: graphgen.rmat(12),
    "road48": lambda: graphgen.road(48),
    "uniform": lambda: graphgen.uniform(3000, 30000),
    "fig1_4": lambda: load("fig1_4.txt")[0],
    "clique_hub": lambda: graphgen.from_edge_list(
        300, [(a, b, 1 + (a * b) % 5) for a in range(40) for b in range(40) if a != b]
        + [(0, v, 2) for v in range(40, 300)] + [(v, (v * 13) % 300, 3) for v in range(40, 300)]),
}
KNOBS = {
    "smem": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=200),
    "smem_und": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=300, sibling_undirected=True),
    "all": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.3,
                   degree_norm=True, degsim_threshold=0.5),
}


def _knobs(gx, kn):
    return gx.Knobs(**{f: getattr(kn, f) for f in kn.__dataclass_fields__})


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
def test_device_transform_matches_oracle(gname, kname):
    import paper_conf_icpp_0001n20_b200 as gx
    raw = GRAPHS[gname]()
    kn = KNOBS[kname]
    G = upload(raw)
    info = G.transform(_knobs(gx, kn))
    assert_same(G.export(), oracle_export(raw, kn), info)


@pytest.mark.parametrize("scale", [16, 18])
@pytest.mark.parametrize("kname", ["smem", "coalesce_smem", "degnorm", "degnorm_wmax", "all"])
def test_device_transform_matches_host_library(scale, kname):
    """Larger RMAT (many triangles, hub rows): device path vs the host-only
    library path, whose transforms are pinned to the oracle on CPU."""
    import paper_conf_icpp_0001n20_b200 as gx
    ctx()
    raw = graphgen.rmat(scale)
    kn = {"smem": T.Knobs(smem=True, cc_threshold=0.5),
          "coalesce_smem": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.4, smem=True,
                                   cc_threshold=0.5),
          "degnorm": T.Knobs(degree_norm=True, degsim_threshold=0.5),
          "degnorm_wmax": T.Knobs(degree_norm=True, degsim_threshold=0.4, added_weight="max"),
          "all": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.4, smem=True, cc_threshold=0.5,
                         degree_norm=True, degsim_threshold=0.4)}[kname]
    G = upload(raw)
    info = G.transform(_knobs(gx, kn))
    H = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    hinfo = H.transform(_knobs(gx, kn))
    a, b = G.export(), H.export()
    for k in ("row_ptr", "col", "w", "edge_added", "slot_to_orig", "slot_kind", "sched", "tile_ptr",
              "tile_members", "tile_centre", "tile_iters"):
        assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), k
    for k in ("n_slots", "n_replicas", "n_holes", "edges_added_coalesce", "edges_added_smem", "edges_added_degnorm",
              "n_subgraphs", "subgraph_vertices"):
        assert info[k] == hinfo[k], k
    assert info["n_subgraphs"] > 0 or info["edges_added_degnorm"] > 0


def test_device_levels_road_grid():
    """High-diameter graph (hundreds of BFS levels): the coalescing
    renumbering from device levels equals the host-only library's."""
    import paper_conf_icpp_0001n20_b200 as gx
    ctx()
    raw = graphgen.road(200)
    kn = T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.4)
    G = upload(raw)
    G.transform(_knobs(gx, kn))
    H = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    H.transform(_knobs(gx, kn))
    a, b = G.export(), H.export()
    for k in ("row_ptr", "col", "slot_to_orig", "slot_kind"):
        assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), k


EXPORT_KEYS = ("row_ptr", "col", "w", "edge_added", "slot_to_orig", "slot_kind", "sched", "tile_ptr",
               "tile_members", "tile_centre", "tile_iters")
INFO_KEYS = ("n_slots", "m_slots", "n_replicas", "n_holes", "edges_added_coalesce", "edges_added_smem",
             "edges_added_degnorm", "n_subgraphs", "subgraph_vertices")

PIPE_GRAPHS = {
    "rmat14": lambda: graphgen.rmat(14),
    "road120": lambda: graphgen.road(120),
    "uniform": lambda: graphgen.uniform(5000, 60000),
    "star_hub": lambda: graphgen.from_edge_list(
        2000, [(0, v, 1 + v % 7) for v in range(1, 2000)] + [(v, (v * 7 + 3) % 2000, 1 + v % 5) for v in range(1, 2000)]
        + [(v, (v + 1) % 2000, 2) for v in range(1, 2000)]),
    "empty_rows": lambda: graphgen.from_edge_list(64, [(1, 2, 3), (2, 5, 1), (5, 1, 4), (9, 2, 2), (40, 41, 9)]),
}
PIPE_KNOBS = {
    # chunk_k = 32: the replica kernel's lane masks use every bit
    "coal_k32": T.Knobs(coalesce=True, chunk_k=32, replicate_threshold=0.1),
    "coal_k4_max": T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.2, added_weight="max"),
    "coal_k8_mean": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.25, added_weight="mean"),
    "coal_degnorm": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.3, degree_norm=True,
                            degsim_threshold=0.5),
    "smem_degnorm": T.Knobs(smem=True, cc_threshold=0.3, degree_norm=True, degsim_threshold=0.6),
    "degnorm_f": T.Knobs(degree_norm=True, degsim_threshold=0.7, degree_target=0.6),
    "all_mean": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.2, smem=True, cc_threshold=0.4,
                        degree_norm=True, degsim_threshold=0.5, added_weight="mean"),
}


@pytest.mark.parametrize("gname", list(PIPE_GRAPHS))
@pytest.mark.parametrize("kname", list(PIPE_KNOBS))
@pytest.mark.parametrize("mode", ["device", "mixed"])
def test_transform_pipelines_agree(gname, kname, mode, monkeypatch):
    """N1: the device-resident pipeline (default with a context) and the round-1
    host pipeline with device helpers (GX_TRANSFORM=mixed) export exactly the
    host-only library's slot graph, which the CPU suite pins to the oracle."""
    import paper_conf_icpp_0001n20_b200 as gx
    ctx()
    if mode == "mixed":
        monkeypatch.setenv("GX_TRANSFORM", "mixed")
    raw = PIPE_GRAPHS[gname]()
    kn = PIPE_KNOBS[kname]
    G = upload(raw)
    info = G.transform(_knobs(gx, kn))
    H = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    hinfo = H.transform(_knobs(gx, kn))
    a, b = G.export(), H.export()
    for k in EXPORT_KEYS:
        assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), k
    for k in INFO_KEYS:
        assert info[k] == hinfo[k], k


def test_device_pipeline_oracle_replicas():
    """A graph where §2 places many replicas (low theta_conn, k = 4): the device
    pipeline's export equals the oracle's element by element."""
    import paper_conf_icpp_0001n20_b200 as gx
    raw = graphgen.rmat(11)
    kn = T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.1)
    G = upload(raw)
    info = G.transform(_knobs(gx, kn))
    assert info["n_replicas"] > 0
    assert_same(G.export(), oracle_export(raw, kn), info)
