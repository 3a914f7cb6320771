"""Multi-GPU host logic on CPU.

* gx_partition_rows: the 1-D partition the library uses -- monotone, aligned
  to the PR window, covers [0, n), (edges + rows) balanced;
* the exchange protocol, run by world_size-2 `gloo` processes: each rank
  relaxes only its own rows, dist is allreduced with MIN, owners rebuild the
  frontier from the distances that dropped, counters are allreduced; PR
  allreduces the owned contrib slices (zero elsewhere).  The per-rank sweep
  here is a plain numpy mirror of the kernel's semantics; the protocol must
  reach the oracle's fixed points exactly (SSSP) / within 1e-9 (PR).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen
from oracle import algos as A
from oracle.graph import from_raw, graph_to_edgelist, sssp_source


@pytest.fixture(scope="module")
def gx():
    from paper_conf_icpp_0001n20_b200 import build
    build.build()
    import paper_conf_icpp_0001n20_b200 as m
    return m


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("gname", ["rmat14", "road64", "tiny"])
def test_partition_properties(gx, P, gname):
    from paper_conf_icpp_0001n20_b200._binding import partition_rows
    raw = {"rmat14": lambda: graphgen.rmat(14), "road64": lambda: graphgen.road(64),
           "tiny": lambda: graphgen.from_edge_list(5, [(0, 1, 1)])}[gname]()
    rp = raw.row_ptr
    n = raw.n
    b = partition_rows(rp, P, 1024)
    assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0)
    assert all(x % 1024 == 0 for x in b[1:-1])
    if n >= 64 * 1024:
        work = np.array([(rp[b[i + 1]] + b[i + 1]) - (rp[b[i]] + b[i]) for i in range(P)])
        tot = rp[n] + n
        # balanced to within one alignment block of work per rank
        assert np.all(np.abs(work - tot / P) <= tot / P * 0.05 + 1024 * 64)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sweep_sssp(g, dist, frontier, lo, hi):
    """numpy mirror of one k_sssp_lb sweep over the rank's rows [lo, hi)."""
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    sel = (src >= lo) & (src < hi) & frontier[src]
    nd = dist[src[sel]] + g.w[sel]
    np.minimum.at(dist, g.col[sel], nd)
    return int(sel.sum())


def _worker_sssp(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_0001n20_b200._binding import partition_rows
    g = from_raw(graphgen.rmat(12))
    b = partition_rows(g.row_ptr, world, 1024)
    lo, hi = int(b[rank]), int(b[rank + 1])
    INF = np.int64(2**32 - 1)
    d = np.full(g.n, INF, dtype=np.int64)
    s = sssp_source(g)
    d[s] = 0
    frontier = np.zeros(g.n, dtype=bool)
    frontier[s] = True
    for it in range(10000):
        old = d.copy()
        _sweep_sssp(g, d, frontier, lo, hi)
        t = torch.from_numpy(d)
        dist.all_reduce(t, op=dist.ReduceOp.MIN)          # the exchange
        d = t.numpy().copy()
        frontier = np.zeros(g.n, dtype=bool)
        frontier[lo:hi] = d[lo:hi] < old[lo:hi]            # owners rebuild their frontier
        cnt = torch.tensor([int(frontier.sum())])
        dist.all_reduce(cnt)                               # global counter
        if int(cnt) == 0:
            break
    out[rank] = (d == np.asarray(A.sssp_dijkstra(graph_to_edgelist(g), s), dtype=np.int64)).all()
    dist.destroy_process_group()


def _worker_pr(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_0001n20_b200._binding import partition_rows
    g = from_raw(graphgen.rmat(12))
    el = graph_to_edgelist(g)
    b = partition_rows(g.row_ptr, world, 1024)
    lo, hi = int(b[rank]), int(b[rank + 1])
    n = g.n
    D = np.bincount(el.src, minlength=n).astype(np.float64)
    x = np.full(n, 1.0 / n)
    contrib = np.where(D > 0, x / np.where(D > 0, D, 1), 0.0)
    dang = x[D == 0].sum()
    for it in range(1000):
        y = np.bincount(el.dst, weights=contrib[el.src], minlength=n)
        own = np.zeros(n, dtype=bool)
        own[lo:hi] = True
        xn = x.copy()
        xn[own] = 0.15 / n + 0.85 * (y[own] + dang / n)
        delta = np.abs(xn[own] - x[own]).sum()
        dng = xn[own & (D == 0)].sum()
        c = np.zeros(n)
        c[own] = np.where(D[own] > 0, xn[own] / np.where(D[own] > 0, D[own], 1), 0.0)
        tc = torch.from_numpy(c)
        dist.all_reduce(tc)                                # owned slices, zero elsewhere
        sc = torch.tensor([delta, dng], dtype=torch.float64)
        dist.all_reduce(sc)
        contrib = tc.numpy().copy()
        dang = float(sc[1])
        x = xn
        if float(sc[0]) < 1e-13:
            break
    xf = np.where(np.arange(n) >= lo, x, 0.0) * (np.arange(n) < hi)
    tx = torch.from_numpy(xf)
    dist.all_reduce(tx)
    want, _ = A.pagerank(el, tol=1e-14)
    out[rank] = float(np.abs(tx.numpy() - want).sum())
    dist.destroy_process_group()


@pytest.mark.parametrize("worker", ["sssp", "pr"])
def test_gloo_world2_exchange_protocol(gx, worker):
    mgr = mp.Manager()
    out = mgr.dict()
    fn = _worker_sssp if worker == "sssp" else _worker_pr
    mp.spawn(fn, args=(2, _free_port(), out), nprocs=2, join=True)
    if worker == "sssp":
        assert out[0] and out[1]
    else:
        assert out[0] < 1e-9 and out[1] < 1e-9


def _coll_worker(rank, world, port, out):
    """One rank driving the hosted-exchange transport (the library's gx_coll_fn
    implementation in the binding) on host buffers, as libgraffix calls it."""
    import ctypes as C
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_0001n20_b200 import hosted_collective
    from paper_conf_icpp_0001n20_b200._binding import (GX_COLL_ALLGATHERV, GX_COLL_ALLREDUCE, GX_COLL_REDUCE_SCATTERV,
                                                       GX_DT_F32, GX_DT_F64, GX_DT_U32, GX_OP_MIN, GX_OP_SUM)
    f = hosted_collective(rank)
    offs = np.array([0, 5, 11], dtype=np.int64)             # unequal slices, as edge-balanced bounds are
    offp = offs.ctypes.data_as(C.POINTER(C.c_int64))
    res = {}
    # allreduce(min) of u32 distances, INF included
    d = np.array([7, 0xFFFFFFFF, 3 + rank, 0xFFFFFFFE, 9 * rank, 1, 2, 3, 4, 5, 6], dtype=np.uint32)
    assert f(GX_COLL_ALLREDUCE, d.ctypes.data, d.size, GX_DT_U32, GX_OP_MIN, None, world, None) == 0
    res["min_u32"] = d.copy()
    # fused scalar allreduce(sum) of f64
    x = np.array([0.25 * (rank + 1), 1e-17, -3.0], dtype=np.float64)
    assert f(GX_COLL_ALLREDUCE, x.ctypes.data, x.size, GX_DT_F64, GX_OP_SUM, None, world, None) == 0
    res["sum_f64"] = x.copy()
    # allgather-v of f32 slices: rank r owns [offs[r], offs[r+1]); other slices hold stale values
    c = np.full(11, 99.0, dtype=np.float32)
    c[offs[rank]:offs[rank + 1]] = np.arange(offs[rank], offs[rank + 1], dtype=np.float32) + 0.5
    assert f(GX_COLL_ALLGATHERV, c.ctypes.data, c.size, GX_DT_F32, GX_OP_SUM, offp, world, None) == 0
    res["gather_f32"] = c.copy()
    # reduce-scatter-v(min) of u32: this rank's slice must hold the min over ranks
    r = np.arange(11, dtype=np.uint32) * (rank + 1) + (10 if rank == 0 else 0)
    assert f(GX_COLL_REDUCE_SCATTERV, r.ctypes.data, r.size, GX_DT_U32, GX_OP_MIN, offp, world, None) == 0
    res["rs_u32"] = r.copy()
    np.savez(os.path.join(out, f"coll{rank}.npz"), **res)
    dist.destroy_process_group()


def test_hosted_exchange_transport_world2(tmp_path):
    """The hosted exchange's transport (include/graffix.h gx_coll_fn, binding
    `hosted_collective`) between two gloo processes on CPU: allreduce min/sum,
    allgather-v with unequal slices, reduce-scatter-v -- the collectives the
    partitioned path issues; the GPU side is tested with two
    processes on one B200 (tests/test_gpu_dist_procs.py)."""
    world = 2
    mp.start_processes(_coll_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True,
                       start_method="spawn")
    offs = [0, 5, 11]
    for rank in range(world):
        z = np.load(tmp_path / f"coll{rank}.npz")
        assert list(z["min_u32"]) == [7, 0xFFFFFFFF, 3, 0xFFFFFFFE, 0, 1, 2, 3, 4, 5, 6]
        assert np.array_equal(z["sum_f64"], np.array([0.75, 2e-17, -6.0]))
        assert np.array_equal(z["gather_f32"], np.arange(11, dtype=np.float32) + 0.5)
        want = np.minimum(np.arange(11) * 1 + 10, np.arange(11) * 2)
        lo, hi = offs[rank], offs[rank + 1]
        assert np.array_equal(z["rs_u32"][lo:hi], want[lo:hi].astype(np.uint32))
