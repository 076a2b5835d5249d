#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 300 python scripts/scan_n.py > gpurun_out/scan_n.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 2 -c 1 -f \
   -o gpurun_out/prof_fill python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_fill_run.log 2>&1
