#!/bin/bash
# GPU parity tests only (PYTEST_ARGS to select)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
