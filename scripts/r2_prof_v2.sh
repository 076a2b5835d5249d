#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_pv2.log; : > $L
timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1
timeout 300 python scripts/repro_fuzz.py 23 300001 5 >> $L 2>&1
REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f \
   -o gpurun_out/r2_pv2_cfg2 python scripts/k1_timing.py cfg2 >> $L 2>&1
REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f \
   -o gpurun_out/r2_pv2_c4e1 python scripts/k1_timing.py cfg4e1 >> $L 2>&1
