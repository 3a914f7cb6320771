#!/bin/bash
# per-kernel launch list + full profile of the PR kernels (tag $1)
TAG=${1:-x}
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_pr_$TAG.csv python tools/prof_run.py --scale 24 --algos pagerank > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_pr_stream|k_pr_update" -s 6 -c 2 -o gpurun_out/prof_pr_$TAG python tools/prof_run.py --scale 24 --algos pagerank > /dev/null 2>&1
GX_PR_VARIANT=2 ncu --set full --clock-control none --import-source on -k regex:"k_pr_stream" -s 3 -c 1 -o gpurun_out/prof_pr2_$TAG python tools/prof_run.py --scale 24 --algos pagerank > /dev/null 2>&1
ls gpurun_out/*$TAG*
