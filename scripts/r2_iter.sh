#!/bin/bash
# one iteration: K1 A/B on full-size epochs (VARIANTS, CASES), then the K1-path parity + dump tests on the in-tree build
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_iter.log; : > $L
for v in ${VARIANTS:-new}; do
  echo "== $v" >> $L
  VE_LIB_PATH=build/libve_$v.so timeout 400 python scripts/k1_timing.py ${CASES:-cfg4e0,cfg4e1} >> $L 2>&1
done
for m in ${CLAIMS:-}; do
  echo "== claim mode $m (in-tree)" >> $L
  VE_CLAIM_MODE=$m timeout 400 python scripts/k1_timing.py ${CCASES:-cfg2} >> $L 2>&1
done
timeout 1500 python -m pytest -q -x -m gpu ${TESTS:-tests/test_gpu_k1_paths.py tests/test_gpu_dump.py tests/test_gpu_parity.py} >> $L 2>&1
echo "tests exit $?" >> $L
