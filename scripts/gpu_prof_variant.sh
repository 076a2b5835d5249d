#!/bin/bash
# ncu full capture of the gemm-epoch k_analyze launch of an alternative build ($1)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
VE_LIB_PATH=$1 timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 3 -c 1 -f \
   -o gpurun_out/prof_variant python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_variant_run.log 2>&1
