"""A/B of an environment knob read when the blocked PageRank layout is built
(e.g. GX_PB_ORDER): for each value a fresh graph (so the layout is rebuilt),
PageRank (pb) to tol 1e-9, best of --reps; exact graphs and knob graphs.

    python tools/pb_layout_ab.py --env GX_PB_ORDER --values 0,1 --cases rmat22,rmat24,c2
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

CASES = {
    "rmat22": (lambda: graphgen.rmat(22), None),
    "rmat24": (lambda: graphgen.rmat(24), None),
    "rmat26": (lambda: graphgen.rmat(26), None),
    "uniform24": (lambda: graphgen.uniform(1 << 24, 1 << 28), None),
    "c2": (lambda: graphgen.rmat(22), dict(coalesce=True, chunk_k=16, replicate_threshold=0.6, merge_op=1)),
    "c2r": (lambda: graphgen.rmat(22), dict(coalesce=True, chunk_k=16, replicate_threshold=2.0)),
    "c3r": (lambda: graphgen.road(4900), dict(coalesce=True, chunk_k=16, replicate_threshold=2.0)),
    "c4": (lambda: graphgen.uniform(1 << 24, 1 << 28), dict(degree_norm=True, degsim_threshold=0.3, degree_target=0.85)),
}
ap = argparse.ArgumentParser()
ap.add_argument("--env", default="GX_PB_ORDER")
ap.add_argument("--values", default="0,1")
ap.add_argument("--cases", default="rmat22,rmat24,c2")
ap.add_argument("--reps", type=int, default=4)
a = ap.parse_args()
ctx = gx.Context(0)
for name in a.cases.split(","):
    mk, kn = CASES[name]
    raw = mk()
    for v in a.values.split(","):
        os.environ[a.env] = v
        G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
        if kn:
            G.transform(gx.Knobs(**kn))
        rs = [G.run("pagerank", mapping="pb", tol=1e-9) for _ in range(a.reps)]
        r = min(rs, key=lambda q: q["loop_ms"])
        print(f"{name} {a.env}={v} loop_ms={r['loop_ms']:.3f} iters={r['iterations']} "
              f"per_sweep_us={1e3 * r['loop_ms'] / max(r['iterations'], 1):.1f}", flush=True)
        G.close()
