#!/bin/bash
# Standard GPU pass: build, gpu tests, bench; optional ncu captures (tag in $1).
TAG=${1:-x}
mkdir -p gpurun_out
python -m paper_conf_icpp_0001n20_b200.build > gpurun_out/build_$TAG.log 2>&1 || { cat gpurun_out/build_$TAG.log; exit 1; }
if [ -z "$NOTEST" ]; then timeout 900 python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-not nothing}" > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log; fi
if [ -z "$NOBENCH" ]; then timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench_$TAG.log 2>&1; tail -c 3000 gpurun_out/bench_$TAG.log; fi
if [ -n "$NCU" ]; then
  ncu --set full --clock-control none --import-source on -k regex:k_pr_stream -s 3 -c 1 -o gpurun_out/prof_pr_$TAG python tools/prof_run.py --scale 24 --algos pagerank > gpurun_out/ncu_pr_$TAG.log 2>&1
  ncu --set full --clock-control none --import-source on -k regex:k_sssp_lb -s 6 -c 2 -o gpurun_out/prof_sssp_$TAG python tools/prof_run.py --scale 24 --algos sssp > gpurun_out/ncu_sssp_$TAG.log 2>&1
fi
true
