#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_uprobe_ab.log; : > $L
for v in ${VARIANTS:-new}; do
  echo "== $v" >> $L
  VE_LIB_PATH=build/libve_$v.so timeout 300 python scripts/units_probe.py 250 0 >> $L 2>&1
done
