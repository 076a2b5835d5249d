#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_i3.log; : > $L
timeout 600 python scripts/k1_timing.py cfg3,cfg2 >> $L 2>&1
timeout 1200 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_cfg34.py tests/test_gpu_k1_paths.py tests/test_gpu_units.py >> $L 2>&1; echo "tests exit $?" >> $L
timeout 700 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f -o gpurun_out/r2_uprof2 python scripts/units_probe.py 250 0 > gpurun_out/r2_uprof2.log 2>&1
python scripts/ncu_lines.py gpurun_out/r2_uprof2.ncu-rep 1964936 60 > gpurun_out/r2_uprof2_lines.txt 2>&1
REPS=1 timeout 700 ncu --set full --clock-control none --import-source on -k regex:k_dense_obj -c 1 -f -o gpurun_out/r2_dobj python scripts/k1_timing.py cfg4e0 > gpurun_out/r2_dobj.log 2>&1
python scripts/ncu_summary.py gpurun_out/r2_dobj.ncu-rep > gpurun_out/r2_dobj_summary.txt 2>&1
