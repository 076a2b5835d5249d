#!/bin/bash
# PROFILING ONLY: K1 time vs shared histogram slots (VE_HS)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/hs.log
for h in 8192 4096 2048 1024 512; do
  echo "== hs $h" >> gpurun_out/hs.log
  VE_HS=$h timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[" | tail -2 >> gpurun_out/hs.log
done
