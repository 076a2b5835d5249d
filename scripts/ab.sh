#!/bin/bash
# A/B timing of alternative libve builds (build/libve_*.so via VE_LIB_PATH), 2 rounds
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for r in 1 2; do
for lib in build/libve_*.so; do
  echo "== $lib" >> gpurun_out/ab.log
  VE_LIB_PATH=$lib timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[" | tail -2 | tr '\n' ' ' >> gpurun_out/ab.log
  echo >> gpurun_out/ab.log
done
done
