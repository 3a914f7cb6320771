#!/bin/bash
# round 1e: LH parity tests + round profile capture (launch list, ncu --set full of k_pr_pb / k_sssp_persist)
python -m paper_conf_icpp_0001n20_b200.build > /dev/null 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -x -q -k "light_heavy" > gpurun_out/pytest_r1e_lh.log 2>&1; tail -2 gpurun_out/pytest_r1e_lh.log
timeout 1200 bash tools/profile_round.sh r1e > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_bench_r1e.csv > gpurun_out/launches_bench_summary_r1e.txt 2>&1
python tools/ncu_summary.py gpurun_out/prof_prpb_r1e.raw.csv gpurun_out/prof_ssspLB_r1e.raw.csv > gpurun_out/ncu_full_summary_r1e.json 2>&1
head -30 gpurun_out/launches_bench_summary_r1e.txt
