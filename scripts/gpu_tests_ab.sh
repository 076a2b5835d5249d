#!/bin/bash
# GPU parity tests of the in-tree build, then A/B timing of build/libve_*.so variants (+ WCLK breakdown if built)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
if [ -f build/libve_wclk.so ]; then
  VE_LIB_PATH=build/libve_wclk.so timeout 300 python scripts/step_timing.py > gpurun_out/wclk.log 2>&1
  mv build/libve_wclk.so build/wclk.so.off
fi
bash scripts/ab.sh
