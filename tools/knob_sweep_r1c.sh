#!/bin/bash
# Knob sweeps with the blocked PR pull in the baselines (round 1c)
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
mkdir -p gpurun_out/knobs_r1c
timeout 600 python tools/knob_sweep.py --config c1 > gpurun_out/knobs_r1c/c1.jsonl 2> gpurun_out/knobs_r1c/c1.err
timeout 1200 python tools/knob_sweep.py --config c2 > gpurun_out/knobs_r1c/c2.jsonl 2> gpurun_out/knobs_r1c/c2.err
timeout 1500 python tools/knob_sweep.py --config c4 > gpurun_out/knobs_r1c/c4.jsonl 2> gpurun_out/knobs_r1c/c4.err
timeout 1500 python tools/knob_sweep.py --config c3 --budgets 0,0.5,1 > gpurun_out/knobs_r1c/c3.jsonl 2> gpurun_out/knobs_r1c/c3.err
python tools/algos_c4.py > gpurun_out/knobs_r1c/c4_algos.jsonl 2> gpurun_out/knobs_r1c/c4_algos.err
wc -l gpurun_out/knobs_r1c/*
