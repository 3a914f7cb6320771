"""Experiment: does a degree-ordered vertex relabelling speed up the exact
sweeps?  Builds permuted copies of RMAT-<scale> on the host (numpy), uploads
each and times SSSP (LB) and PageRank (tol 1e-9).

    python tools/relabel_exp.py --scale 24
"""
import argparse
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402


def permute(rp, col, w, rank):
    """new id of old v = rank[v]; rows keep their internal order."""
    n = len(rp) - 1
    order = np.empty(n, dtype=np.int64)
    order[rank] = np.arange(n)
    deg = np.diff(rp)
    nrp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(deg[order], out=nrp[1:])
    # edge index of new row r, position j = rp[order[r]] + j
    src_start = np.repeat(rp[:-1][order] - nrp[:-1], deg[order])
    idx = np.arange(len(col), dtype=np.int64) + src_start
    return nrp, rank[col[idx]].astype(np.int32), w[idx]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--orders", default="none,out,outin,in,random")
    ap.add_argument("--algos", default="sssp,pagerank")
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    raw = graphgen.rmat(a.scale)
    rp = raw.row_ptr.astype(np.int64)
    col = raw.col.astype(np.int64)
    w = raw.w
    n = len(rp) - 1
    outd = np.diff(rp)
    ind = np.bincount(col, minlength=n)
    ctx = gx.Context(0)
    for o in a.orders.split(","):
        t0 = time.time()
        if o == "none":
            prp, pcol, pw = rp, raw.col, w
        else:
            key = {"out": outd, "in": ind, "outin": outd + ind,
                   "random": np.random.default_rng(1).permutation(n)}[o]
            ordv = np.argsort(-key, kind="stable")
            rank = np.empty(n, dtype=np.int64)
            rank[ordv] = np.arange(n)
            prp, pcol, pw = permute(rp, col, w, rank)
        tp = time.time() - t0
        G = gx.Graph.upload(ctx, prp, pcol, pw)
        res = {}
        for al, mp, kw in (("sssp", "lb", {}), ("pagerank", "lb", {"tol": 1e-9}), ("pagerank", "pb", {"tol": 1e-9})):
            if al not in a.algos.split(","):
                continue
            rs = [G.run(al, mapping=mp, **kw) for _ in range(a.reps)]
            b = min(rs, key=lambda r: r["loop_ms"])
            res[al + "_" + mp] = (round(b["loop_ms"], 3), b["iterations"], b["edges_scanned"])
        print(f"order={o} permute_s={tp:.1f} " + " ".join(f"{k}={v}" for k, v in res.items()), flush=True)
        G.close()


if __name__ == "__main__":
    main()
