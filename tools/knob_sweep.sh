#!/bin/bash
python -m paper_conf_icpp_0001n20_b200.build > /dev/null
mkdir -p gpurun_out/knobs
timeout 600 python tools/knob_sweep.py --config c1 > gpurun_out/knobs/c1.jsonl 2> gpurun_out/knobs/c1.err
timeout 900 python tools/knob_sweep.py --config c2 --scale-down > gpurun_out/knobs/c2s.jsonl 2> gpurun_out/knobs/c2s.err
timeout 900 python tools/knob_sweep.py --config c4 --scale-down > gpurun_out/knobs/c4s.jsonl 2> gpurun_out/knobs/c4s.err
timeout 900 python tools/knob_sweep.py --config c3 --scale-down --budgets 0,0.5,1,5 > gpurun_out/knobs/c3s.jsonl 2> gpurun_out/knobs/c3s.err
wc -l gpurun_out/knobs/*
