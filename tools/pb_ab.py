"""A/B of the PageRank sweep mappings (LB windowed SELL vs the blocked pull).

    python tools/pb_ab.py --graph rmat --scale 24 --maps lb,pb --reps 3
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=24)
ap.add_argument("--graph", default="rmat")
ap.add_argument("--maps", default="lb,pb")
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--schedules", default="async")
ap.add_argument("--knobs", default="", help="all | smem | coalesce | degnorm (transform before timing)")
ap.add_argument("--aware", action="store_true", help="algorithm-aware merge (GX_MERGE_MIN)")
a = ap.parse_args()
raw = {"rmat": lambda: graphgen.rmat(a.scale), "road": lambda: graphgen.road(a.scale),
       "uniform": lambda: graphgen.uniform(1 << a.scale, 16 << a.scale)}[a.graph]()
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
if a.knobs:
    kw = {"all": dict(coalesce=True, chunk_k=16, replicate_threshold=0.6, smem=True, cc_threshold=0.5,
                      degree_norm=True, degsim_threshold=0.3),
          "smem": dict(smem=True, cc_threshold=0.5), "coalesce": dict(coalesce=True, chunk_k=16, replicate_threshold=0.6),
          "degnorm": dict(degree_norm=True, degsim_threshold=0.3)}[a.knobs]
    if a.aware:
        kw["merge_op"] = 1
    t0 = time.time()
    info = G.transform(gx.Knobs(**kw))
    print(f"transform {a.knobs}: {time.time() - t0:.1f} s, {info}", flush=True)
ref = None
for mp in a.maps.split(","):
    t0 = time.time()
    G.run("pagerank", mapping=mp, tol=1e-9)        # builds the layout
    print(f"{mp}: first run (incl. layout build) {time.time() - t0:.2f} s", flush=True)
    for sch in a.schedules.split(","):
        if mp == "pb" and sch != "async":
            continue
        for rep in range(a.reps):
            r = G.run("pagerank", mapping=mp, tol=1e-9, profile=True, pr_schedule=sch)
            x = G.download("rank")
            if ref is None:
                ref = x
            print(f"{mp:3s} {sch:6s} iters={r['iterations']:3d} loop={r['loop_ms']:7.2f} ms "
                  f"sweep={r['sweep_ms'] / max(r['sweep_launches'], 1) * 1e3:7.1f} us/launch "
                  f"per-it={r['sweep_ms'] / max(r['iterations'], 1) * 1e3:7.1f} us "
                  f"GB/s={r['sweep_bytes'] / (r['sweep_ms'] * 1e-3) / 1e9:7.0f} delta={r['last_delta']:.2e} "
                  f"L1(vs first)={np.abs(x - ref).sum():.2e} used={r['mapping_used']}", flush=True)
