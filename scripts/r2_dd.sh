#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; L=gpurun_out/r2_dd.log; : > $L
timeout 900 python -m pytest -x -q tests/test_gpu_cfg5.py tests/test_gpu_shard.py tests/test_gpu_parity.py tests/test_gpu_dyadic.py tests/test_gpu_fits2.py >> $L 2>&1; echo "tests exit $?" >> $L
timeout 900 python bench.py --no-e2e --no-cpu --steps 3 --warmup 2 > gpurun_out/r2_dd_bench.json 2>> $L; echo "bench exit $?" >> $L
