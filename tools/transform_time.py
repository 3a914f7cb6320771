"""Time the Graffix transforms per pipeline (N1): the device-resident one
(default with a context), the round-1 host pipeline with device helpers
(GX_TRANSFORM=mixed) and, optionally, host only (GX_TRANSFORM=host); checks
that the exports are identical.  Per-phase times with GX_TRANSFORM_TRACE=1.

    python tools/transform_time.py --graph rmat24 --knobs all3 --modes device,mixed
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

MAKE = {"rmat22": lambda: graphgen.rmat(22), "rmat24": lambda: graphgen.rmat(24), "rmat26": lambda: graphgen.rmat(26),
        "uniform24": lambda: graphgen.uniform(1 << 24, 1 << 28), "road4900": lambda: graphgen.road(4900),
        "road1024": lambda: graphgen.road(1024)}
# the C2-C5 knob settings (composition R34 for all3)
KNOBS = {
    "coalesce": dict(coalesce=True, chunk_k=16, replicate_threshold=0.6),
    "smem": dict(smem=True, cc_threshold=0.5),
    "degnorm": dict(degree_norm=True, degsim_threshold=0.3, degree_target=0.85),
    "all3": dict(coalesce=True, chunk_k=16, replicate_threshold=0.6, smem=True, cc_threshold=0.5,
                 degree_norm=True, degsim_threshold=0.3, degree_target=0.85),
}
KEYS = ("row_ptr", "col", "w", "edge_added", "slot_to_orig", "slot_kind", "sched", "tile_ptr", "tile_members",
        "tile_centre", "tile_iters")

ap = argparse.ArgumentParser()
ap.add_argument("--graph", default="rmat24")
ap.add_argument("--knobs", default="all3")
ap.add_argument("--modes", default="device,mixed")
ap.add_argument("--no-compare", action="store_true")
a = ap.parse_args()
raw = MAKE[a.graph]()
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
n, m = raw.n, raw.m
del raw
base = None
for mode in a.modes.split(","):
    os.environ["GX_TRANSFORM"] = mode
    t0 = time.time()
    info = G.transform(gx.Knobs(**KNOBS[a.knobs]))
    wall = time.time() - t0
    same = None
    if not a.no_compare:
        ex = G.export()
        if base is None:
            base = {k: np.asarray(ex[k]).copy() for k in KEYS}
        else:
            same = all(np.array_equal(base[k], np.asarray(ex[k])) for k in KEYS)
        del ex
    print(json.dumps({"graph": a.graph, "n": n, "m": m, "knobs": a.knobs, "mode": mode,
                      "transform_ms": info["transform_ms"], "wall_s": wall, "n_slots": info["n_slots"],
                      "m_slots": info["m_slots"], "replicas": info["n_replicas"],
                      "added": [info["edges_added_coalesce"], info["edges_added_smem"], info["edges_added_degnorm"]],
                      "extra_space_pct": info["extra_space_pct"], "same_as_first": same}), flush=True)
G.close()
