#!/bin/bash
# bench + ncu launch list + ncu full capture of k_analyze (run under gpurun)
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench exit $?" >> gpurun_out/bench.err
if [ "${NCU:-1}" = "1" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_run.log 2>&1
echo "ncu launches exit $?" >> gpurun_out/bench.err
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_analyze -s 2 -c 1 -f \
   -o gpurun_out/prof_analyze python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full_run.log 2>&1
echo "ncu full exit $?" >> gpurun_out/bench.err
fi
