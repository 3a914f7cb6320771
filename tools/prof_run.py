"""Minimal driver for ncu: build a workload graph, run the sweeps once or twice.

    python tools/prof_run.py --scale 24 --algos sssp,pagerank [--reps 1] [--knobs exact]
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
ap.add_argument("--algos", default="sssp,pagerank")
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--mapping", default="lb")
a = ap.parse_args()
raw = graphgen.rmat(a.scale) if a.graph == "rmat" else graphgen.road(a.scale)
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
for _ in range(a.reps):
    for al in a.algos.split(","):
        r = G.run(al, mapping=a.mapping, use_graphs=False, check_every=4)
        print(al, r)
