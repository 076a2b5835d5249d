#!/bin/bash
# A/B of build/libve_*.so variants on the report path (report[1] wall time), 2 rounds
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for r in 1 2; do
for lib in build/libve_*.so; do
  echo "== $lib" >> gpurun_out/ab.log
  VE_TIMING=1 VE_LIB_PATH=$lib timeout 300 python scripts/step_timing.py 2>&1 | grep "report\[\|diff\[\|analyze\[" | tail -5 | tr '\n' ' ' >> gpurun_out/ab.log
  echo >> gpurun_out/ab.log
done
done
