#!/bin/bash
for f in paper_conf_icpp_0001n20_b200/libgraffix.so paper_conf_icpp_0001n20_b200/libgraffix_w*.so; do
  echo -n "$(basename $f): "; GX_LIB_PATH=$PWD/$f python tools/prof_run.py --scale 24 --algos pagerank --reps 2 2>&1 | grep -o "'loop_ms': [0-9.]*" | tr '\n' ' '; echo
done
