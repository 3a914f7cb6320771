"""C3 road grid: PageRank / SSSP with and without the §3 knob, per-phase times (profile mode).

    python tools/road_smem_pr.py --side 4900
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
import paper_conf_icpp_0001n20_b200 as gx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--side", type=int, default=4900)
ap.add_argument("--maps", default="lb,pb")
a = ap.parse_args()
raw = graphgen.road(a.side)
ctx = gx.Context(0)
keys = ["iterations", "loop_ms", "sweep_ms", "smem_ms", "merge_ms", "sweep_launches", "mapping_used", "last_delta"]
for knob in ["exact", "smem"]:
    G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
    if knob == "smem":
        t0 = time.time()
        info = G.transform(gx.Knobs(smem=True, cc_threshold=0.5))
        print(f"transform: {time.time() - t0:.1f} s subgraphs={info['n_subgraphs']} members={info['subgraph_vertices']}",
              flush=True)
    for algo, maps in [("pagerank", a.maps.split(",")), ("sssp", ["lb"])]:
        for mp in maps:
            G.run(algo, mapping=mp, tol=1e-9)
            for prof in [False, True]:
                r = G.run(algo, mapping=mp, tol=1e-9, profile=prof)
                print(knob, algo, mp, "profile" if prof else "timed", {k: r.get(k) for k in keys}, flush=True)
    G.close()
