#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
for h in 256 128 64 32 16; do
  echo -n "PR_HEAVY $h: "; GX_PR_HEAVY=$h python tools/prof_run.py --scale 24 --algos pagerank --reps 2 2>&1 | grep -o "'iterations': [0-9]*\|'loop_ms': [0-9.]*" | tr '\n' ' '; echo
done
