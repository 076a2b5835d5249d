#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
free -g > gpurun_out/r2_bench.err; nproc >> gpurun_out/r2_bench.err
timeout 1500 python bench.py > gpurun_out/r2_bench.json 2>> gpurun_out/r2_bench.err
echo "bench exit $?" >> gpurun_out/r2_bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r2_bench_ref.json 2>> gpurun_out/r2_bench.err
echo "ref exit $?" >> gpurun_out/r2_bench.err
