"""Per-iteration timing of the persistent SSSP loop (GX_SSSP_PTRACE=1 makes
k_sssp_persist record globaltimer / edges / frontier size per iteration).

    GX_SSSP_PTRACE=1 python tools/sssp_ptrace.py --graph rmat24 [--knob degnorm]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--graph", default="rmat24")
ap.add_argument("--knob", default="exact")
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
mk = {"rmat24": lambda: graphgen.rmat(24), "rmat22": lambda: graphgen.rmat(22),
      "uniform24": lambda: graphgen.uniform(1 << 24, 1 << 28), "rmat26": lambda: graphgen.rmat(26)}[a.graph]
raw = mk()
ctx = gx.Context(0)
G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
if a.knob == "degnorm":
    G.transform(gx.Knobs(degree_norm=True, degsim_threshold=0.3))
for i in range(a.reps):
    print(f"== rep {i}", file=sys.stderr, flush=True)
    r = G.run("sssp", mapping="lb")
    print(f"rep {i}: loop_ms={r['loop_ms']:.3f} iters={r['iterations']} edges={r['edges_scanned']}", flush=True)
