#!/bin/bash
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_dyadic.py -x -q > gpurun_out/gpu_dy.log 2>&1; echo "exit $?" >> gpurun_out/gpu_dy.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "exit $?" >> gpurun_out/smoke.log
timeout 1200 python bench.py --steps 5 --warmup 3 --no-cfg5 --no-cfg34 --no-cpu --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?" >> gpurun_out/bench.err
bash scripts/gpu_dy_prof.sh
