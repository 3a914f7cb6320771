"""Per-iteration SSSP trace (GX_SSSP_TRACE, profile mode): frontier sizes,
near-far threshold and sweep-kernel time, for several bucket widths.

    python tools/sssp_trace.py --scale 24 --deltas auto,0,12,25,50,100
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
ap.add_argument("--deltas", default="auto")
ap.add_argument("--trace", action="store_true")
a = ap.parse_args()
raw = graphgen.rmat(a.scale) if a.graph == "rmat" else graphgen.road(a.scale)
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
G.run("sssp")
for dl in a.deltas.split(","):
    if dl == "auto":
        os.environ.pop("GX_SSSP_DELTA", None)
    else:
        os.environ["GX_SSSP_DELTA"] = dl
    best = min((G.run("sssp") for _ in range(3)), key=lambda r: r["loop_ms"])
    print(f"delta={dl} loop_ms={best['loop_ms']:.3f} iters={best['iterations']} edges={best['edges_scanned']}",
          flush=True)
    if a.trace:
        os.environ["GX_SSSP_TRACE"] = "1"
        G.run("sssp", profile=True)
        os.environ.pop("GX_SSSP_TRACE")
    sys.stderr.flush()
