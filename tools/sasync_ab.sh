set -x
export VARIANTS="-DGX_PB_SASYNC=0;-DGX_PB_SASYNC=1 -DGX_PB_SDEPTH=5;-DGX_PB_SASYNC=1 -DGX_PB_SDEPTH=3;-DGX_PB_SASYNC=1 -DGX_PB_SDEPTH=4"
bash tools/pb_variants.sh > gpurun_out/sasync_ab.txt 2>&1
GX_NVCC_EXTRA="-DGX_PB_SASYNC=1" python -m paper_conf_icpp_0001n20_b200.build --force > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "pagerank or pr or pb" > gpurun_out/sasync_pytest.txt 2>&1; tail -3 gpurun_out/sasync_pytest.txt
cat gpurun_out/sasync_ab.txt
