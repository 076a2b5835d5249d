#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 300 python scripts/cfg5_timing.py > gpurun_out/cfg5_timing.log 2>&1
VE_TIMING=2 timeout 300 python scripts/cfg5_timing.py 0 1000 2000 > gpurun_out/cfg5_timing_stages.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cfg5_launches.csv \
  python scripts/cfg5_timing.py 0 1000 2000 > gpurun_out/cfg5_ncu_run.log 2>&1
