#!/bin/bash
# bench + GPU tests + ncu launch list of the bench command + a full capture of each cfg4 k_analyze epoch
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; E=gpurun_out/r2_bench.err; : > $E
timeout 2400 python -m pytest -q -m gpu tests/ > gpurun_out/r2_gpu_tests.log 2>&1; echo "tests exit $?" >> $E
timeout 1500 python bench.py > gpurun_out/r2_bench.json 2>> $E; echo "bench exit $?" >> $E
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file gpurun_out/r2_bench_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-extra --no-cfg5 \
   > gpurun_out/r2_ncu_launch_run.log 2>&1; echo "ncu launches exit $?" >> $E
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 2 -c 2 -f \
   -o gpurun_out/r2_bench_k1 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-extra --no-cfg5 \
   > gpurun_out/r2_ncu_full_run.log 2>&1; echo "ncu full exit $?" >> $E
