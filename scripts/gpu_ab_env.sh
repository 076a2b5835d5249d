#!/bin/bash
# A/B of build variants plus the base build under environment knobs
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
bash scripts/ab.sh
for hs in 4096 2048; do
  echo "== base VE_HS=$hs" >> gpurun_out/ab.log
  VE_HS=$hs VE_LIB_PATH=build/libve_base.so timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[" | tail -2 | tr '\n' ' ' >> gpurun_out/ab.log
  echo >> gpurun_out/ab.log
done
