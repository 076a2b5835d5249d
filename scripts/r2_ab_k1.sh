#!/bin/bash
# A/B of K1 build variants (build/libve_<v>.so) on full-size epochs: VARIANTS, CASES
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_ab_k1.log; : > $L
for v in ${VARIANTS:-base}; do
  echo "== $v" >> $L
  VE_LIB_PATH=build/libve_$v.so timeout 400 python scripts/k1_timing.py ${CASES:-cfg4e0,cfg4e1} >> $L 2>&1
done
