#!/bin/bash
# A/B of build/libve_*.so variants: cfg2 analyze (step_timing) and cfg4 analyze / report (cfg34_timing)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for lib in build/libve_*.so; do
  echo "== $lib" >> gpurun_out/ab.log
  VE_LIB_PATH=$lib timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[\|report\[" | tail -4 | tr '\n' ' ' >> gpurun_out/ab.log
  echo >> gpurun_out/ab.log
  VE_TIMING=1 VE_LIB_PATH=$lib timeout 600 python scripts/cfg34_timing.py ${CFG34:-cfg4} 2>&1 | grep "==\|analyze\|dense_flush\|report" >> gpurun_out/ab.log
done
