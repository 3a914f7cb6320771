for u in ${SEGUS:-4 2 8}; do
  GX_NVCC_EXTRA="-DGX_PB_SEGU=$u" python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
  echo "SEGU=$u"; timeout 200 python tools/pb_ab.py --scale 24 --maps pb --reps 2 2>&1 | grep async
done
