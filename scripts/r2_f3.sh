#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_f3.log; : > $L
timeout 900 python -m pytest -x -q tests/test_gpu_temporal.py >> $L 2>&1; echo "exit $?" >> $L
