#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
VE_TIMING=2 timeout 300 python scripts/step_timing.py > gpurun_out/step_timing.log 2>&1
bash scripts/ab.sh
if [ "${NCU:-0}" = "1" ]; then
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 3 -c 1 -f \
   -o gpurun_out/prof_gemm python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_run.log 2>&1
fi
