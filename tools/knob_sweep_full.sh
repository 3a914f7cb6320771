#!/bin/bash
# Full-size knob sweeps (BASELINE.json configs C2-C4; C1 is already full size).
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
mkdir -p gpurun_out/knobs_full
timeout 600 python tools/knob_sweep.py --config c1 > gpurun_out/knobs_full/c1.jsonl 2> gpurun_out/knobs_full/c1.err
timeout 1500 python tools/knob_sweep.py --config c2 > gpurun_out/knobs_full/c2.jsonl 2> gpurun_out/knobs_full/c2.err
timeout 1500 python tools/knob_sweep.py --config c4 > gpurun_out/knobs_full/c4.jsonl 2> gpurun_out/knobs_full/c4.err
timeout 1500 python tools/knob_sweep.py --config c3 --budgets 0,0.1,0.5,1,2,5 > gpurun_out/knobs_full/c3.jsonl 2> gpurun_out/knobs_full/c3.err
wc -l gpurun_out/knobs_full/*
