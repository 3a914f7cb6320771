#!/bin/bash
# Round profile capture: launch list of the bench command (cold, serialised)
# + ncu --set full of the dominant kernels.  Output in gpurun_out/prof_$1*.
TAG=${1:-r1}
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-knobs > gpurun_out/bench_under_ncu_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_pr_pb" -s 5 -c 1 -o gpurun_out/prof_prpb_$TAG \
    python tools/prof_run.py --scale 24 --algos pagerank --mapping pb > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_sssp_persist" -s 1 -c 1 -o gpurun_out/prof_ssspLB_$TAG \
    python tools/prof_run.py --scale 24 --algos sssp --reps 2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_sssp_pb_" -s 2 -c 2 -o gpurun_out/prof_ssspPB_$TAG \
    python tools/prof_run.py --scale 24 --algos sssp --reps 2 > /dev/null 2>&1
for f in gpurun_out/prof_prpb_$TAG gpurun_out/prof_ssspLB_$TAG gpurun_out/prof_ssspPB_$TAG; do
  ncu -i $f.ncu-rep --page details --csv > $f.details.csv 2>/dev/null
  ncu -i $f.ncu-rep --page raw --csv > $f.raw.csv 2>/dev/null
done
ls -la gpurun_out/*$TAG*
