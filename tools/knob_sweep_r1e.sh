#!/bin/bash
# Knob sweeps with the blocked PR pull in the baselines (round 1e, at HEAD)
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
mkdir -p gpurun_out/knobs_r1e
timeout 600 python tools/knob_sweep.py --config c1 > gpurun_out/knobs_r1e/c1.jsonl 2> gpurun_out/knobs_r1e/c1.err
timeout 1200 python tools/knob_sweep.py --config c2 > gpurun_out/knobs_r1e/c2.jsonl 2> gpurun_out/knobs_r1e/c2.err
timeout 1500 python tools/knob_sweep.py --config c4 > gpurun_out/knobs_r1e/c4.jsonl 2> gpurun_out/knobs_r1e/c4.err
timeout 1500 python tools/knob_sweep.py --config c3 --budgets 0,0.5,1 > gpurun_out/knobs_r1e/c3.jsonl 2> gpurun_out/knobs_r1e/c3.err
python tools/algos_c4.py > gpurun_out/knobs_r1e/c4_algos.jsonl 2> gpurun_out/knobs_r1e/c4_algos.err
wc -l gpurun_out/knobs_r1e/*
