#!/bin/bash
# A/B of k_pb_init_val variants through the bench (PR loop incl. the initial scatter)
IFS=';' read -ra VS <<< "${VARIANTS:--DGX_PB_SASYNC=0 -DGX_PB_INIT_MINB=1;-DGX_PB_INIT_MINB=1;-DGX_PB_INIT_MINB=2}"
for v in "${VS[@]}"; do
  GX_NVCC_EXTRA="$v" python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
  for r in 1 2; do
    timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('[$v]', 'step %.3f ms' % d['ms_per_step'], 'pr loop %.3f ms' % d['per_algo']['pagerank']['loop_ms'], 'sssp %.3f' % d['per_algo']['sssp']['loop_ms'])"
  done
done
python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "pagerank or pr or pb" 2>&1 | tail -1
