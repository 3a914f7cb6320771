#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
for v in 0 4 2 6; do
  echo "variant $v"; GX_PR_VARIANT=$v python tools/prof_run.py --scale 24 --algos pagerank --reps 2 2>&1 | grep -o "'iterations': [0-9]*\|'loop_ms': [0-9.]*" | tr '\n' ' '; echo
done
