#!/bin/bash
# per-kernel launch list (ncu gpu__time_duration) of k1_timing on CASES (REPS=1), in-tree build
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
for c in ${LCASES:-cfg4e1}; do
REPS=1 timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2_launch_$c.csv python scripts/k1_timing.py $c > gpurun_out/r2_launch_$c.log 2>&1
python scripts/launch_shares.py gpurun_out/r2_launch_$c.csv > gpurun_out/r2_launch_${c}_shares.txt 2>&1
done
