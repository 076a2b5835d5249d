#!/bin/bash
# ncu full capture of the gemm-epoch k_analyze launch (+ launch list)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-f1 --no-cfg5 --no-cfg34 > gpurun_out/ncu_launch_run.log 2>&1
echo "ncu launches exit $?" > gpurun_out/prof.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 3 -c 1 -f \
   -o gpurun_out/prof_gemm python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-f1 --no-cfg5 --no-cfg34 > gpurun_out/ncu_full_run.log 2>&1
echo "ncu full exit $?" >> gpurun_out/prof.err
