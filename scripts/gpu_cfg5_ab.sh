#!/bin/bash
# cfg5 per-kernel costs under env knobs (dense pool off, smaller K1 shared table)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
K="0 200 400 1000 1400 2000 3600"
timeout 300 python scripts/cfg5_timing.py $K > gpurun_out/c5_base.log 2>&1
VE_DENSE_BUDGET=0 timeout 300 python scripts/cfg5_timing.py $K > gpurun_out/c5_nodense.log 2>&1
VE_HS=512 timeout 300 python scripts/cfg5_timing.py $K > gpurun_out/c5_hs512.log 2>&1
VE_DENSE_BUDGET=0 VE_HS=512 timeout 300 python scripts/cfg5_timing.py $K > gpurun_out/c5_both.log 2>&1
