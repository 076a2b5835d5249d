#!/bin/bash
# ncu source-level capture of k_analyze2 on cfg4 epoch 0 / 1 (full size) + per-line tables
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_pl.log; : > $L
for c in ${CASES:-cfg4e0 cfg4e1}; do
REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-k_analyze2} -c 1 -f \
   -o gpurun_out/r2_pl_$c python scripts/k1_timing.py $c >> $L 2>&1
echo "$c exit $?" >> $L
U=1; [ $c = cfg4e0 ] && U=33554432; [ $c = cfg4e1 ] && U=29360128; python scripts/ncu_lines.py gpurun_out/r2_pl_$c.ncu-rep $U 90 > gpurun_out/r2_pl_${c}_lines.txt 2>&1
python scripts/ncu_summary.py gpurun_out/r2_pl_$c.ncu-rep > gpurun_out/r2_pl_${c}_summary.txt 2>&1
done
