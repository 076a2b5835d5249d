#!/bin/bash
# round-2 probe: per-phase timing of cfg3/cfg4 + ncu launch list of one cfg4 epoch-0 analyze+report
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_probe.log
timeout 600 python scripts/cfg34_timing.py both >> gpurun_out/r2_probe.log 2>&1
echo "timing exit $?" >> gpurun_out/r2_probe.log
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,sm__cycles_active.max,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg4_launches.csv \
   python scripts/cfg34_timing.py cfg4 > gpurun_out/r2_ncu_run.log 2>&1
echo "ncu exit $?" >> gpurun_out/r2_probe.log
