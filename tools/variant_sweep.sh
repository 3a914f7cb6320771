#!/bin/bash
# Build compile-time variants of libgraffix.so and time RMAT-24 PR / SSSP with each.
#   VARIANTS="base: u16:-DGX_PR_U=16 minb6:-DGX_PR_MINB=6" tools/variant_sweep.sh [build|run|all]
# (GX_BUILD_OUT / GX_BUILD_OBJ / GX_NVCC_EXTRA: paper_conf_icpp_0001n20_b200/build.py; GX_LIB_PATH: _binding.py)
# build_var/ is git-ignored but ships to the GPU box, so variants can be built here and run there.
MODE=${1:-all}
mkdir -p gpurun_out build_var
if [ "$MODE" != run ]; then
  for v in ${VARIANTS}; do
    name=${v%%:*}; flags=${v#*:}; flags=${flags//,/ }   # several flags: comma-separated
    GX_BUILD_OUT=build_var/lib_$name.so GX_BUILD_OBJ=build_var/obj_$name GX_NVCC_EXTRA="$flags" \
      python -m paper_conf_icpp_0001n20_b200.build > build_var/build_$name.log 2>&1 || { echo "build $name failed"; tail build_var/build_$name.log; }
  done
fi
if [ "$MODE" != build ]; then
  for v in ${VARIANTS}; do
    name=${v%%:*}
    echo "== $name ${v#*:}"
    GX_LIB_PATH=build_var/lib_$name.so python tools/relabel_exp.py --scale ${SCALE:-24} --orders none --algos ${ALGOS:-pagerank} --reps ${REPS:-3}
  done
fi
