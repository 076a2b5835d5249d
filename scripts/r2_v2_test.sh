#!/bin/bash
# v2 K1: quick parity + A/B timing of thread-count variants and v1
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_v2.log; : > $L
timeout 900 python -m pytest -x -q tests/test_gpu_k1_paths.py -k "fuzz5_both or cfg1_both" >> $L 2>&1
echo "k1 paths exit $?" >> $L
timeout 900 python -m pytest -x -q tests/test_gpu_parity.py >> $L 2>&1
echo "parity exit $?" >> $L
for lib in paper_conf_asplos_zhouhmm022_b200/libve.so build/libve_t384.so build/libve_t256.so; do
  echo "== $lib" >> $L
  VE_LIB_PATH=$lib timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
done
echo "== v1" >> $L
VE_K1=1 timeout 300 python scripts/k1_timing.py cfg2,cfg4e0,cfg4e1,cfg3 >> $L 2>&1
