"""N4: Graffix layouts under a virtual-node-splitting engine (Tigr-style, the
paper's second workload P@11477-11746, on our own kernels).  SSSP time with
the thread-per-vertex mapping (TPV), virtual node splitting (VNS, K edges per
virtual node) and the edge-balanced LB kernel, in exact mode and with the §2
and §4 knobs; speedup of each knob over exact under the SAME mapping.

    python tools/vns_sweep.py --graph rmat --scale 22 [--ks 4,8,16]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--graph", default="rmat")
ap.add_argument("--scale", type=int, default=22)
ap.add_argument("--ks", default="4,8,16")
a = ap.parse_args()
raw = {"rmat": lambda: graphgen.rmat(a.scale), "road": lambda: graphgen.road(a.scale),
       "uniform": lambda: graphgen.uniform(1 << a.scale, 16 << a.scale)}[a.graph]()
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
knobs = [("exact", None), ("coalesce t0.6", gx.Knobs(coalesce=True)),
         ("degnorm t0.3", gx.Knobs(degree_norm=True)), ("degnorm t0.5", gx.Knobs(degree_norm=True, degsim_threshold=0.5)),
         ("coalesce+degnorm", gx.Knobs(coalesce=True, degree_norm=True))]
base = {}
for kname, kn in knobs:
    t0 = time.time()
    G.transform(kn)
    tr = time.time() - t0
    arms = [("tpv", None), ("lb", None)] + [("vns", k) for k in a.ks.split(",")]
    for mp, k in arms:
        if k:
            os.environ["GX_VNS_K"] = k
        G.run("sssp", mapping=mp)
        best = min((G.run("sssp", mapping=mp) for _ in range(3)), key=lambda r: r["loop_ms"])
        key = (mp, k)
        if kname == "exact":
            base[key] = best["loop_ms"]
        print(json.dumps({"graph": f"{a.graph}{a.scale}", "knob": kname, "mapping": mp, "K": k,
                          "loop_ms": best["loop_ms"], "iterations": best["iterations"],
                          "edges": best["edges_scanned"], "transform_s": tr,
                          "speedup_same_mapping": base[key] / best["loop_ms"]}), flush=True)
