#!/bin/bash
# bench.py twice: default hist capacity and VE_BENCH_HCAP=${HCAP_B:-4194304}
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_a.json 2> gpurun_out/bench_a.err
VE_BENCH_HCAP=${HCAP_B:-4194304} timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-f1 > gpurun_out/bench_b.json 2> gpurun_out/bench_b.err
VE_TIMING=2 VE_BENCH_HCAP=${HCAP_B:-4194304} timeout 300 python scripts/step_timing.py > gpurun_out/step_timing_b.log 2>&1
