"""A/B timing of PR sweep variants on one graph (env GX_PR_KERNEL etc. per arm).

    python tools/ab_pr.py --scale 24 --arms GX_PR_KERNEL=1 GX_PR_KERNEL=2 --reps 3
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=24)
ap.add_argument("--graph", default="rmat")
ap.add_argument("--arms", nargs="+", default=["GX_PR_KERNEL=1", "GX_PR_KERNEL=2"])
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--algo", default="pagerank")
a = ap.parse_args()
raw = {"rmat": lambda: graphgen.rmat(a.scale), "road": lambda: graphgen.road(a.scale),
       "uniform": lambda: graphgen.uniform(1 << a.scale, 16 << a.scale)}[a.graph]()
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
G.run(a.algo, mapping="lb")
res = {arm: [] for arm in a.arms}
for _ in range(a.reps):
    for arm in a.arms:
        kw = {}
        for kv in arm.split(","):
            k, v = kv.split("=")
            if k.islower():
                kw[k] = int(v) if v.lstrip("-").isdigit() else v   # run() keyword, e.g. pr_schedule=async
            else:
                os.environ[k] = v
        r = G.run(a.algo, mapping="lb", profile=True, check_every=1, **kw)
        res[arm].append((r["loop_ms"], r["iterations"], r["sweep_ms"] / max(1, r["iterations"])))
        for kv in arm.split(","):
            if not kv.split("=")[0].islower():
                os.environ.pop(kv.split("=")[0], None)
for arm, v in res.items():
    best = min(v)
    print(f"{arm:40s} loop_ms {best[0]:8.3f} iters {best[1]:4d} sweep_ms/iter {min(x[2] for x in v):.4f}")
