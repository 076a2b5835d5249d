#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
bash scripts/ab.sh
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 2 -c 1 -f \
   -o gpurun_out/prof_fill python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_fill_run.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 3 -c 1 -f \
   -o gpurun_out/prof_gemm python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_run.log 2>&1
