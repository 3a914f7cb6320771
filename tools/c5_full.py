"""C5 at full size: RMAT-26 (the paper's rmat26, P@35940; 67.1M vertices, 1.07B
edges) with all three Graffix techniques combined (§2 k=16 theta_conn=0.6, §3
theta_cc=0.5 budget 1%, §4 theta_d=0.3 f=0.85; composition R34), on one GPU:
transform time and extra space (Table 5 analogue, P@40874), SSSP / PageRank
time per mapping against the exact run on the untransformed graph (speedup
vs the same mapping and vs the best exact kernel) and the inaccuracy of the
knob run (R40, P@40990).  One JSON line.

    python tools/c5_full.py [--scale 26]
"""
import argparse
import json
import os

# the exact-mode layouts of every mapping are resident when the transform runs:
# release them first (the device pipeline needs the memory, include/graffix.h)
os.environ.setdefault("GX_TRANSFORM_FREE_LAYOUTS", "1")
import resource
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402


def inacc(a, e, inf=None):
    a = np.asarray(a, np.float64)
    e = np.asarray(e, np.float64)
    ok = np.ones(a.shape, bool) if inf is None else (a != inf) & (e != inf)
    return float(100 * np.abs(a[ok] - e[ok]).sum() / max(np.abs(e[ok]).sum(), 1e-300))


ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=26)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--merge", default="mean", choices=["mean", "aware"],
                help="§2.4 confluence: the paper's mean (P@28609) or the algorithm-aware one (P@28421, R54)")
a = ap.parse_args()
t0 = time.time()
raw = graphgen.rmat(a.scale)
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
del raw
gen_s = time.time() - t0
maps = {"sssp": ["lb", "tpv"], "pagerank": ["pb", "lb", "tpv"]}


def timed(algo, mp):
    kw = {"tol": 1e-9} if algo == "pagerank" else {}
    rs = [G.run(algo, mapping=mp, **kw) for _ in range(a.reps)]
    r = min(rs, key=lambda q: q["loop_ms"])
    return {"ms": r["loop_ms"], "iterations": r["iterations"], "edges": r["edges_scanned"]}


ex = {al: {mp: timed(al, mp) for mp in mps} for al, mps in maps.items()}
G.run("sssp", mapping="lb")
de = G.download("dist").copy()
G.run("pagerank", mapping="pb", tol=1e-9)
xe = G.download("rank").copy()
t1 = time.time()
info = G.transform(gx.Knobs(coalesce=True, chunk_k=16, replicate_threshold=0.6, merge_op=int(a.merge == "aware"),
                            smem=True, cc_threshold=0.5,
                            added_edge_budget=-1, degree_norm=True, degsim_threshold=0.3, degree_target=0.85))
tr_s = time.time() - t1
kn = {al: {mp: timed(al, mp) for mp in mps} for al, mps in maps.items()}
G.run("sssp", mapping="lb")
da = G.download("dist")
G.run("pagerank", mapping="lb", tol=1e-9)
xa = G.download("rank")
out = {"config": f"C5: RMAT-{a.scale}, all three techniques (k16 theta_conn 0.6 {a.merge} merge | theta_cc 0.5 budget 1% | theta_d 0.3 f 0.85)",
       "n": G.n, "m": G.m, "gen_upload_s": gen_s, "transform_s": tr_s, "transform_info": info,
       "exact": ex, "knobs": kn,
       "speedup_vs_best_exact": {al: min(v["ms"] for v in ex[al].values()) / min(v["ms"] for v in kn[al].values())
                                 for al in maps},
       "speedup_same_mapping": {al: {mp: ex[al][mp]["ms"] / kn[al][mp]["ms"] for mp in maps[al]} for al in maps},
       "inaccuracy_pct": {"sssp": inacc(da, de, 0xFFFFFFFF), "pagerank": inacc(xa, xe)},
       "host_peak_rss_gb": resource.getrusage(resource.RUSAGE_SELF).ru_maxrss / 2**20}
print(json.dumps(out))
