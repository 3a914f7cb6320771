"""Parity of the production transforms (libgraffix host C++) with the oracle.

Both sides implement §2/§3/§4 from the paper independently (readings R1-R44);
the library's exported slot graph must equal the oracle's element by element:
slot count, slot CSR (rows sorted by destination, R11), weights, added-edge
kinds, slot -> vertex map, slot kinds, the §4 warp schedule and the §3 tiles.
Runs on CPU through gx_graph_create_host (no device needed)."""
import numpy as np
import pytest

import graphgen
from golden_io import load
from oracle import transform as T
from oracle.graph import from_raw


@pytest.fixture(scope="module")
def gx():
    from paper_conf_icpp_0001n20_b200 import build
    build.build()
    import paper_conf_icpp_0001n20_b200 as m
    return m


def lib_transform(gx, raw, kn: T.Knobs):
    G = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    info = G.transform(gx.Knobs(**{f: getattr(kn, f) for f in kn.__dataclass_fields__}))
    return G.export(), info


def oracle_export(raw, kn: T.Knobs):
    g = from_raw(raw)
    tg = T.transform(g, kn)
    rp, col, w, ad = tg.csr()
    tiles = tg.tiles
    tp = [0]
    mem = []
    for c, members, t in tiles:
        mem.extend(members)
        tp.append(len(mem))
    return dict(n_slots=tg.n_slots, row_ptr=rp, col=col, w=w, edge_added=ad, slot_to_orig=tg.slot_to_orig,
                slot_kind=tg.slot_kind, sched=tg.sched, tile_ptr=np.asarray(tp), tile_members=np.asarray(mem),
                tile_centre=np.asarray([c for c, _, _ in tiles]), tile_iters=np.asarray([t for _, _, t in tiles]),
                info=tg.info)


def assert_same(lib, ora, info):
    assert lib["n_slots"] == ora["n_slots"]
    for k in ("row_ptr", "col", "w", "edge_added", "slot_to_orig", "slot_kind", "sched", "tile_ptr",
              "tile_members", "tile_centre", "tile_iters"):
        a = np.asarray(lib[k]).astype(np.int64)
        b = np.asarray(ora[k]).astype(np.int64)
        assert a.shape == b.shape, (k, a.shape, b.shape)
        assert np.array_equal(a, b), (k, np.nonzero(a != b)[0][:10])
    oi = ora["info"]
    for k in ("n_replicas", "n_holes", "edges_added_coalesce", "edges_added_smem", "edges_added_degnorm",
              "n_subgraphs", "subgraph_vertices"):
        assert info[k] == oi[k], (k, info[k], oi[k])


KNOBS = {
    "exact": T.Knobs(),
    "coal_k16_t06": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.6),
    "coal_k4_t03": T.Knobs(coalesce=True, chunk_k=4, replicate_threshold=0.3),
    "coal_renumber_only": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=2.0),
    "smem": T.Knobs(smem=True, cc_threshold=0.5),
    "smem_t03_b50": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=50, smem_max_nodes=16),
    "degnorm": T.Knobs(degree_norm=True, degsim_threshold=0.3),
    "degnorm_t06": T.Knobs(degree_norm=True, degsim_threshold=0.6, degree_target=0.7),
    "all": T.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.4, smem=True, cc_threshold=0.4,
                   degree_norm=True, degsim_threshold=0.5),
    # N3 variants: alternative added-edge weights (P@34692), undirected sibling edges (P@29950)
    "all_wmax": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.4,
                        degree_norm=True, degsim_threshold=0.5, added_weight="max"),
    "all_wmean": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.4,
                         degree_norm=True, degsim_threshold=0.5, added_weight="mean"),
    "smem_undirected": T.Knobs(smem=True, cc_threshold=0.4, sibling_undirected=True),
    "smem_undirected_wmax": T.Knobs(smem=True, cc_threshold=0.3, added_edge_budget=80, sibling_undirected=True,
                                    added_weight="max"),
}

GRAPHS = {
    "rmat10": lambda: graphgen.rmat(10),
    "road20": lambda: graphgen.road(20),
    "uniform": lambda: graphgen.uniform(700, 5000),
    "fig1_4": lambda: load("fig1_4.txt")[0],
}


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
def test_transform_parity(gx, gname, kname):
    raw = GRAPHS[gname]()
    lib, info = lib_transform(gx, raw, KNOBS[kname])
    assert_same(lib, oracle_export(raw, KNOBS[kname]), info)


def test_transform_parity_rmat12_all(gx):
    raw = graphgen.rmat(12)
    kn = T.Knobs(coalesce=True, smem=True, degree_norm=True)
    lib, info = lib_transform(gx, raw, kn)
    assert_same(lib, oracle_export(raw, kn), info)


def test_fig1_4_through_library(gx):
    raw, meta, ex = load("fig1_4.txt")
    lib, info = lib_transform(gx, raw, T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.6))
    assert lib["n_slots"] == 24 and info["n_replicas"] == 1
    rp = lib["row_ptr"]
    row6 = sorted(lib["col"][rp[6]:rp[7]].tolist())
    assert row6 == [16, 17, 18, 19, 20, 21]            # moved {16,18,20,21} + added {17,19} (P@27117-27600)
    assert lib["slot_kind"][7] == 2 and rp[8] == rp[7]  # hole 7 stays empty


def test_knob_validation(gx):
    raw = graphgen.rmat(6)
    G = gx.Graph.host_only(raw.row_ptr, raw.col, raw.w)
    for bad in (dict(chunk_k=0), dict(chunk_k=33), dict(cc_threshold=1.5), dict(degree_target=0.0),
                dict(smem_max_nodes=1), dict(degsim_threshold=-0.1)):
        with pytest.raises(gx.GraffixError) as e:
            G.transform(gx.Knobs(coalesce=True, **bad))
        assert e.value.status == 1
    with pytest.raises(gx.GraffixError) as e:
        G.run("sssp")
    assert e.value.status == 2
