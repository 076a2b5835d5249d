#!/bin/bash
# quick GPU check: parity tests + per-call step timing
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
VE_TIMING=2 timeout 300 python scripts/step_timing.py > gpurun_out/step_timing.log 2>&1
