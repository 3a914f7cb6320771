"""The 1-D partitioned path with REAL processes: two ranks,
two processes sharing one GPU, each with its own gx_ctx (gx_ctx_create_hosted)
whose collectives go through torch.distributed over gloo.  Everything but the
transport is the library's partitioned code: rank-local layouts (rows [lo,hi)
only), the sweeps, the reduce-scatter / allgather / fused scalar exchanges
and the device-side stop decisions.  SSSP must equal the oracle's Dijkstra
bit for bit, PageRank be within L1 1e-6 of the oracle, BC (source-parallel)
within rel 1e-9 of Brandes, SCC labels equal Tarjan's and the MST weight
Kruskal's (each rank sweeping its share of the edges) -- for exact mode and a
transformed graph with replica groups, §3 tiles and §4 padding (the
allreduce + merge branch)."""
import json
import os
import socket

import numpy as np
import pytest

import graphgen
from oracle import algos as A
from oracle import transform as T
from oracle.graph import from_raw, graph_to_edgelist, sssp_source

pytestmark = pytest.mark.gpu

KNOBS = {
    "exact": None,
    "all": T.Knobs(coalesce=True, chunk_k=8, replicate_threshold=0.3, smem=True, cc_threshold=0.3,
                   degree_norm=True, degsim_threshold=0.5),
}
GRAPHS = {"rmat13": lambda: graphgen.rmat(13), "road48": lambda: graphgen.road(48)}
BC_SOURCES = [0, 7, 100, 1000, 2047]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, gname, kname, out_dir):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_icpp_0001n20_b200 as gx
    torch.cuda.set_device(0)
    ctx = gx.Context.hosted(0, rank, world)
    raw = GRAPHS[gname]()
    G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    kn = KNOBS[kname]
    if kn:
        G.transform(gx.Knobs(**{f: getattr(kn, f) for f in kn.__dataclass_fields__}))
    a = G.run("sssp", mapping="lb", check_every=4)
    dist_ = G.download("dist")
    b = G.run("pagerank", mapping="lb", tol=1e-11, max_iters=5000, check_every=4)
    rank_ = G.download("rank")
    # BC source-parallel: 5 sources split 3 / 2 over the ranks, one allreduce(sum)
    c = G.run("bc", bc_sources=BC_SOURCES)
    np.save(os.path.join(out_dir, f"bc{rank}.npy"), G.download("bc"))
    # SCC (colour rounds, max over the ranks) and MST (Borůvka, min proposals over the ranks)
    d = G.run("scc")
    np.save(os.path.join(out_dir, f"scc{rank}.npy"), G.download("label"))
    e = G.run("mst")
    mst_w = int(G.download("mst_weight"))
    np.save(os.path.join(out_dir, f"dist{rank}.npy"), dist_)
    np.save(os.path.join(out_dir, f"rank{rank}.npy"), rank_)
    with open(os.path.join(out_dir, f"info{rank}.json"), "w") as f:
        json.dump({"sssp": a, "pr": b, "bc": c, "scc": d, "mst": e, "mst_w": mst_w}, f)
    G.close()
    ctx.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("gname", list(GRAPHS))
@pytest.mark.parametrize("kname", list(KNOBS))
def test_two_process_partitioned_run(tmp_path, gname, kname):
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    world = 2
    mp.start_processes(_worker, args=(world, _free_port(), gname, kname, str(tmp_path)), nprocs=world,
                       join=True, start_method="spawn")
    raw = GRAPHS[gname]()
    g = from_raw(raw)
    kn = KNOBS[kname]
    el = T.transform(g, kn).logical() if kn else graph_to_edgelist(g)
    want_d = A.sssp_dijkstra(el, sssp_source(g))
    want_x, _ = A.pagerank(el, tol=1e-14)
    infos = [json.load(open(tmp_path / f"info{r}.json")) for r in range(world)]
    want_bc = A.bc_brandes(el, BC_SOURCES)
    want_scc = A.scc_tarjan(el)
    want_mst = A.mst_kruskal(el)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"dist{r}.npy"), want_d), r
        assert np.abs(np.load(tmp_path / f"rank{r}.npy") - want_x).sum() <= 1e-6, r
        assert infos[r]["sssp"]["converged"] == 1 and infos[r]["pr"]["converged"] >= 1
        got_bc = np.load(tmp_path / f"bc{r}.npy")
        assert np.allclose(got_bc, want_bc, rtol=1e-9, atol=1e-9 * max(1.0, float(np.abs(want_bc).max()))), r
        assert np.array_equal(np.load(tmp_path / f"scc{r}.npy").astype(np.int64), want_scc), r
        assert infos[r]["mst_w"] == want_mst, r
    # each rank swept its share of the logical edges
    assert infos[0]["scc"]["iterations"] == infos[1]["scc"]["iterations"]
    assert infos[0]["mst"]["iterations"] == infos[1]["mst"]["iterations"]
    # the two ranks took the same decisions (same iteration counts) and split the relaxations
    assert infos[0]["sssp"]["iterations"] == infos[1]["sssp"]["iterations"]
    assert infos[0]["pr"]["iterations"] == infos[1]["pr"]["iterations"]
    assert infos[0]["pr"]["edges_scanned"] + infos[1]["pr"]["edges_scanned"] == \
        infos[0]["pr"]["iterations"] * G_m_slots(raw, kn)


def G_m_slots(raw, kn):
    g = from_raw(raw)
    tg = T.transform(g, kn) if kn else T.identity(g)
    return sum(len(r) for r in tg.rows)
