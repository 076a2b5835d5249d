#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_full_tests.log; : > $L
timeout 2400 python -m pytest -q -m gpu tests/ >> $L 2>&1
echo "tests exit $?" >> $L
VE_LIB_PATH=build/libve_k512.so timeout 300 python scripts/k1_timing.py cfg4e0,cfg4e1,cfg3 >> $L 2>&1
