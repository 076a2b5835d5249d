#!/bin/bash
# full round check on the GPU box: parity tests, smoke, bench, ncu launch list + full capture of k_analyze
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python -m pytest tests/ -x -q -m gpu ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1; echo "exit $?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "exit $?" >> gpurun_out/smoke.log
timeout 900 python bench.py --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?" >> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref exit $?" >> gpurun_out/bench_ref.err
if [ "${NCU:-1}" = "1" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-f1 --no-cfg5 --no-cfg34 > gpurun_out/ncu_launch_run.log 2>&1
echo "ncu launches exit $?" >> gpurun_out/bench.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 3 -c 1 -f \
   -o gpurun_out/prof_gemm python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-f1 --no-cfg5 --no-cfg34 > gpurun_out/ncu_full_run.log 2>&1
echo "ncu full exit $?" >> gpurun_out/bench.err
fi
