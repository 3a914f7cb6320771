#!/bin/bash
# ncu --set full of one kernel launch: tools/ncu_one.sh TAG KERNEL_REGEX SKIP -- prof_run args
TAG=$1; K=$2; S=$3; shift 4
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 -o gpurun_out/prof_$TAG python tools/prof_run.py "$@" > gpurun_out/prof_$TAG.log 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page details --csv > gpurun_out/prof_$TAG.details.csv
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv > gpurun_out/prof_$TAG.source.csv 2>/dev/null
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/prof_$TAG.raw.csv 2>/dev/null
tail -2 gpurun_out/prof_$TAG.log
