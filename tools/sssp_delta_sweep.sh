#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
for dl in 0 1000 400 200 100 50 25 12; do
  echo -n "delta $dl: "; GX_SSSP_DELTA=$dl python tools/prof_run.py --scale 24 --algos sssp --reps 2 2>&1 | grep -o "'iterations': [0-9]*\|'loop_ms': [0-9.]*\|'edges_scanned': [0-9]*" | tail -3 | tr '\n' ' '; echo
done
echo -n "default: "; python tools/prof_run.py --scale 24 --algos sssp --reps 2 2>&1 | grep -o "'iterations': [0-9]*\|'loop_ms': [0-9.]*\|'edges_scanned': [0-9]*" | tail -3 | tr '\n' ' '; echo
