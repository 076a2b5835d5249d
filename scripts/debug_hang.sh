#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
for n in 65536 32768 100003 300001 1000000; do
  echo "== n=$n" >> gpurun_out/dbg.log
  timeout 120 python scripts/debug_stage.py 2 $n >> gpurun_out/dbg.log 2>&1
  echo "rc $?" >> gpurun_out/dbg.log
done
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1
echo "exit $?" >> gpurun_out/gpu_tests.log
