#!/bin/bash
# round-2 evidence: GPU tests, bench line (+ reference arm), ncu launch list of the bench step, full capture of both K1 epochs
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out; E=gpurun_out/r2f.err; : > $E
timeout 1500 python -m pytest -q -m gpu tests/ > gpurun_out/r2f_gpu_tests.log 2>&1; echo "tests exit $?" >> $E
timeout 1500 python bench.py > gpurun_out/r2f_bench.json 2>> $E; echo "bench exit $?" >> $E
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r2f_bench_ref.json 2>> $E; echo "ref exit $?" >> $E
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file gpurun_out/r2f_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-extra --no-cfg5 \
   > gpurun_out/r2f_ncu_launch_run.log 2>&1; echo "ncu launches exit $?" >> $E
python scripts/launch_shares.py gpurun_out/r2f_launches.csv > gpurun_out/r2f_launch_shares.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 2 -c 2 -f \
   -o gpurun_out/r2f_k1 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-extra --no-cfg5 \
   > gpurun_out/r2f_ncu_full_run.log 2>&1; echo "ncu full exit $?" >> $E
python scripts/ncu_summary.py gpurun_out/r2f_k1.ncu-rep > gpurun_out/r2f_k1_summary.txt 2>&1
