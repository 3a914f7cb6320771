#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
python tools/prof_run.py --scale 24 --algos sssp,pagerank --reps 2 2>&1 | grep -o "^[a-z]*\|'iterations': [0-9]*\|'loop_ms': [0-9.]*\|'edges_scanned': [0-9]*" | tr '\n' ' '; echo
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$1.csv python tools/prof_run.py --scale 24 --algos sssp,pagerank > /dev/null 2>&1
