#!/bin/bash
# A/B of compile-time PB variants: VARIANTS="-DGX_PB_CPT=2 -DGX_PB_NST=3" (one quoted flag set per word group, ';' separated)
IFS=';' read -ra VS <<< "${VARIANTS:- }"
for v in "${VS[@]}"; do
  GX_NVCC_EXTRA="$v" python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
  echo "variant [$v]"; timeout 200 python tools/pb_ab.py --scale ${SCALE:-24} --maps pb --reps 2 2>&1 | grep async
done
