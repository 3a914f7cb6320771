#!/bin/bash
# quick timings: RMAT-24 exact SSSP/PR and RMAT-20 coalesced (renumbered) SSSP LB
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
python tools/prof_run.py --scale 24 --algos sssp,pagerank --reps 2 2>&1 | grep -o "^[a-z]*\|'iterations': [0-9]*\|'loop_ms': [0-9.]*\|'edges_scanned': [0-9]*" | tr '\n' ' '; echo
python - <<'PY'
import sys; sys.path.insert(0, '.')
import graphgen, paper_conf_icpp_0001n20_b200 as gx
raw = graphgen.rmat(20); ctx = gx.Context(0); G = gx.Graph.upload(ctx, raw.row_ptr, raw.col, raw.w)
for kn in (None, gx.Knobs(coalesce=True, replicate_threshold=2.0)):
    G.transform(kn)
    print("coalesce" if kn else "exact", [round(G.run("sssp", mapping="lb")["loop_ms"], 3) for _ in range(3)])
PY
