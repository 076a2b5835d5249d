#!/bin/bash
# A/B timing of alternative libve builds (VE_LIB_PATH)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for lib in paper_conf_asplos_zhouhmm022_b200/libve.so build/libve_384.so; do
  echo "== $lib" >> gpurun_out/ab.log
  VE_LIB_PATH=$lib timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[" | tail -2 >> gpurun_out/ab.log
done
timeout 900 python -m pytest tests/ -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
