#!/bin/bash
# GPU tests + default bench line (sanity of HEAD on a fresh box)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_check.log; : > $L
timeout 1800 python -m pytest -q -m gpu tests/ >> $L 2>&1
echo "tests exit $?" >> $L
timeout 1200 python bench.py > gpurun_out/r2_check_bench.json 2>> $L
echo "bench exit $?" >> $L
