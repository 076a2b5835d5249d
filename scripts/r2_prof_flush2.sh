#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
VE_K1=1 REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_dense_obj -c 1 -f \
   -o gpurun_out/r2_prof_flush2 python scripts/k1_timing.py cfg4e0 > /dev/null 2>&1
REPS=1 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_active.avg,sm__cycles_active.max --clock-control none --csv --log-file gpurun_out/r2_flush_launches2.csv python scripts/k1_timing.py cfg2,cfg3 > /dev/null 2>&1
