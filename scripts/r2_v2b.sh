#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_v2b.log; : > $L
timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1; echo "plain exit $?" >> $L
timeout 600 compute-sanitizer --tool synccheck --print-limit 10 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1; echo "synccheck exit $?" >> $L
for lib in paper_conf_asplos_zhouhmm022_b200/libve.so build/libve_t384.so; do
  echo "== $lib" >> $L
  VE_LIB_PATH=$lib timeout 300 python scripts/repro_fuzz.py 4 300001 >> $L 2>&1
  VE_LIB_PATH=$lib timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
done
