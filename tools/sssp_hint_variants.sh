#!/bin/bash
# A/B of compile-time SSSP variants (RMAT-24 exact): VARIANTS="-DGX_SSSP_RP_EF=1;-DGX_SSSP_SU=8"
IFS=';' read -ra VS <<< "${VARIANTS:- }"
for v in "${VS[@]}"; do
  GX_NVCC_EXTRA="$v" python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
  echo "variant [$v]"; timeout 200 python tools/sssp_trace.py --scale 24 --deltas auto,25 2>&1 | grep delta
done
