#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 1 -c 1 -f \
   -o gpurun_out/prof_c5 python scripts/cfg5_timing.py 1000 > gpurun_out/ncu_c5_run.log 2>&1
echo "exit $?" >> gpurun_out/ncu_c5_run.log
