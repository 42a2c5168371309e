#!/bin/bash
# One GPU session: parity tests, bench lines, ncu launch list + full capture of the top kernels.
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 300 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; tail -3 gpurun_out/bench_c2.err
timeout 300 python bench.py --workload C3 --no-cpu-baseline > gpurun_out/bench_c3.json 2>&1
timeout 300 python bench.py --workload C4 --no-cpu-baseline --steps 200 > gpurun_out/bench_c4.json 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 30 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:coarse -s 4 -c 1 -o gpurun_out/prof_c2_coarse python bench.py --steps 6 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fine_rows -s 2 -c 1 -o gpurun_out/prof_c4_fine python bench.py --workload C4 --steps 4 --warmup 2 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
ls -la gpurun_out
