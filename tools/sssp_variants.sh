#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
for f in 2.0 0.05 0.02 0.005 0; do
  echo "dense_frac $f"; GX_DENSE_FRAC=$f python tools/prof_run.py --scale 24 --algos sssp --reps 2 2>&1 | grep -o "'iterations': [0-9]*\|'loop_ms': [0-9.]*\|'edges_scanned': [0-9]*" | tr '\n' ' '; echo
done
