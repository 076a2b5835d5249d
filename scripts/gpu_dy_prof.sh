#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,smsp__warps_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_registers --clock-control none --csv -k regex:k_dy --log-file gpurun_out/dy_launches.csv python scripts/dy_prof.py > gpurun_out/dy_prof.log 2>&1
echo "exit $?" >> gpurun_out/dy_prof.log
