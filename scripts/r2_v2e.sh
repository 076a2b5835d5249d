#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_v2e.log; : > $L
timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1
timeout 300 python scripts/repro_fuzz.py 23 300001 5 >> $L 2>&1
timeout 300 python scripts/repro_fuzz.py 26 8400017 >> $L 2>&1
timeout 600 python -m pytest -x -q tests/test_gpu_parity.py tests/test_gpu_cfg34.py >> $L 2>&1
timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
VE_K1=1 timeout 300 python scripts/k1_timing.py cfg2,cfg4e0 >> $L 2>&1
