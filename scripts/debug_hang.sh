#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; rm -f gpurun_out/dbg.log
python -c "import torch; torch.zeros(1).cuda()" > /dev/null 2>&1
for args in "4 150000"; do
  echo "== $args" >> gpurun_out/dbg.log
  start=$(date +%s)
  timeout 300 python scripts/debug_stage.py $args > gpurun_out/dbg_one.log 2>&1
  echo "rc $? secs $(( $(date +%s) - start ))" >> gpurun_out/dbg.log
  grep -v "^diff" gpurun_out/dbg_one.log | tail -12 >> gpurun_out/dbg.log
done
