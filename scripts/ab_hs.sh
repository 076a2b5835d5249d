#!/bin/bash
# A/B of K1's shared value-table size (VE_HS) on the cfg2 step
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for r in 1 2; do
for hs in 8192 4096 2048 1024; do
  echo "== VE_HS=$hs" >> gpurun_out/ab.log
  VE_HS=$hs timeout 300 python scripts/step_timing.py 2>/dev/null | grep "analyze\[\|report\[\|diff\[" | tail -5 | tr '\n' ' ' >> gpurun_out/ab.log
  echo >> gpurun_out/ab.log
done
done
