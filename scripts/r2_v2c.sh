#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_v2c.log; : > $L
for lib in paper_conf_asplos_zhouhmm022_b200/libve.so build/libve_t384.so; do
  echo "== $lib" >> $L
  VE_LIB_PATH=$lib timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1
  VE_LIB_PATH=$lib timeout 300 python scripts/repro_fuzz.py 23 300001 5 >> $L 2>&1
  VE_LIB_PATH=$lib timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
done
REPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_analyze2 -c 1 -f \
   -o gpurun_out/r2_pv2c_cfg2 python scripts/k1_timing.py cfg2 >> /dev/null 2>&1
