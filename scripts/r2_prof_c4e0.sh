#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
VE_LIB_PATH=build/libve_t384.so REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f \
   -o gpurun_out/r2_pv2c_c4e0 python scripts/k1_timing.py cfg4e0 > /dev/null 2>&1
VE_LIB_PATH=build/libve_t384.so REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f \
   -o gpurun_out/r2_pv2c_c4e1 python scripts/k1_timing.py cfg4e1 > /dev/null 2>&1
