#!/bin/bash
# cfg5 records half: GPU parity + the full bench line
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cfg5.py -x -q > gpurun_out/gpu_cfg5.log 2>&1; echo "exit $?" >> gpurun_out/gpu_cfg5.log
timeout 1200 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?" >> gpurun_out/bench.err
