python -m paper_conf_icpp_0001n20_b200.build > /dev/null 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -x -q -k "sssp" > gpurun_out/pytest_lh1.log 2>&1; tail -3 gpurun_out/pytest_lh1.log
GX_SSSP_LH=0 python tools/sssp_trace.py --scale 24 --deltas auto,50 > gpurun_out/lh1_off.txt 2>&1
GX_SSSP_LH=1 python tools/sssp_trace.py --scale 24 --deltas auto,12,18,35,50,75,100 > gpurun_out/lh1_on.txt 2>&1
cat gpurun_out/lh1_off.txt gpurun_out/lh1_on.txt
