"""PageRank for each value of one environment knob (GX_PB_SYM, ...): sweeps to
tol, time, and the fixed-point residual ||x - F(x)||_1 of each result (bound
r / (1 - d) on the distance to the PageRank vector; F = the PR map of
PAPER.md P@36969, R35).  (Round 2 used it as pr_omega.py for GX_PR_OMEGA.)

    python tools/pr_env_sweep.py --scale 24 --env GX_PB_SYM --values 0,1
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402


def residual(rp, col, x, d=0.85):
    n = len(rp) - 1
    deg = np.diff(rp)
    src = np.repeat(np.arange(n), deg)
    c = np.where(deg > 0, x / np.maximum(deg, 1), 0.0)
    y = np.bincount(col, weights=c[src], minlength=n)
    fx = (1 - d) / n + d * (y + x[deg == 0].sum() / n)
    return float(np.abs(x - fx).sum())


ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=24)
ap.add_argument("--env", default="GX_PB_SYM")
ap.add_argument("--values", default="0,1")
ap.add_argument("--mapping", default="pb")
a = ap.parse_args()
raw = graphgen.rmat(a.scale)
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
ex = G.export()
rp, col = ex["row_ptr"], ex["col"]
for om in a.values.split(","):
    os.environ[a.env] = om
    runs = [G.run("pagerank", tol=1e-9, mapping=a.mapping) for _ in range(3)]
    r = min(runs, key=lambda q: q["loop_ms"])
    x = G.download("rank")
    res = residual(rp, col, x)
    print(f"{a.env}={om} sweeps={r['iterations']} loop_ms={r['loop_ms']:.2f} last_delta={r['last_delta']:.3e} "
          f"converged={r['converged']} residual={res:.3e} bound={res / 0.15:.3e} mass={x.sum():.12f}", flush=True)
