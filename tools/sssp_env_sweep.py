"""Time SSSP (LB mapping, persistent loop) for each value of one GX_SSSP_*
environment knob on generated graphs; checks the distances stay identical.

    python tools/sssp_env_sweep.py --env GX_SSSP_DENSE --values 0,0.5,0.3 --graphs rmat24,uniform24
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

MAKE = {"rmat24": lambda: graphgen.rmat(24), "rmat22": lambda: graphgen.rmat(22), "rmat26": lambda: graphgen.rmat(26),
        "uniform24": lambda: graphgen.uniform(1 << 24, 1 << 28), "road4900": lambda: graphgen.road(4900), "road1024": lambda: graphgen.road(1024)}
ap = argparse.ArgumentParser()
ap.add_argument("--env", required=True)
ap.add_argument("--values", required=True)
ap.add_argument("--graphs", default="rmat24,uniform24,road4900")
ap.add_argument("--reps", type=int, default=4)
a = ap.parse_args()
ctx = gx.Context(0)
for gname in a.graphs.split(","):
    raw = MAKE[gname]()
    G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    del raw
    base = None
    for v in a.values.split(","):
        os.environ[a.env] = v
        rs = [G.run("sssp", mapping="lb") for _ in range(a.reps)]
        r = min(rs, key=lambda q: q["loop_ms"])
        d = G.download("dist")
        if base is None:
            base = d.copy()
        print(f"{gname} {a.env}={v} loop_ms={r['loop_ms']:.3f} iters={r['iterations']} "
              f"dense_it={r['dense_iterations']} edges={r['edges_scanned']} same={np.array_equal(d, base)}", flush=True)
    G.close()
