#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_san.log; : > $L
timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1; echo "plain exit $?" >> $L
for tool in synccheck memcheck; do
  echo "== $tool" >> $L
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1
  echo "$tool exit $?" >> $L
done
