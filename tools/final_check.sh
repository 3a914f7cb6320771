#!/bin/bash
# end-of-session check: build() as the driver runs it, full GPU suite, smoke(), default bench, reference arm
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/final_build.log 2>&1 || { tail -20 gpurun_out/final_build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/final_pytest.log 2>&1; tail -2 gpurun_out/final_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; tail -2 gpurun_out/final_smoke.log
timeout 600 python bench.py > gpurun_out/final_bench.log 2>&1; tail -c 600 gpurun_out/final_bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.log 2>&1; tail -c 400 gpurun_out/final_bench_ref.log
