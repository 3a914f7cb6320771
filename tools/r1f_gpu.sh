#!/bin/bash
# r1f: full GPU suite, default bench, then the round profile (launch list + ncu --set full of k_pr_pb / k_sssp_persist)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r1f_build.log 2>&1 || { tail -20 gpurun_out/r1f_build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r1f_pytest.log 2>&1; tail -2 gpurun_out/r1f_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1f_smoke.log 2>&1; tail -1 gpurun_out/r1f_smoke.log
timeout 600 python bench.py > gpurun_out/r1f_bench.log 2>&1; tail -c 300 gpurun_out/r1f_bench.log
timeout 1500 bash tools/profile_round.sh r1f > /dev/null 2>&1; ls gpurun_out | grep r1f
