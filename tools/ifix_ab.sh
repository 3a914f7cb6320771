#!/bin/bash
# A/B: phase (1) fixed-point conversion by F2I.U64 (GX_PB_IFIX=0) vs integer instructions (1)
VARIANTS="-DGX_PB_IFIX=0;-DGX_PB_IFIX=1;-DGX_PB_IFIX=0;-DGX_PB_IFIX=1" bash tools/pb_variants.sh
python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "pagerank or pr or pb" 2>&1 | tail -1
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | cut -c1-400
