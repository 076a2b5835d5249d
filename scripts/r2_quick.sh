#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_quick.log; : > $L
timeout 900 python -m pytest -x -q tests/test_gpu_shard.py tests/test_gpu_parity.py tests/test_gpu_cfg34.py >> $L 2>&1
echo "tests exit $?" >> $L
timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
