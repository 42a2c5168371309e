#!/bin/bash
# Round profile capture (one GPU): launch lists + full captures of the dominant kernels.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for W in C2 C4; do
  timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_$W.csv python bench.py --workload $W --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
done
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:coarse -s 3 -c 1 -o gpurun_out/full_c2_coarse \
  python bench.py --workload C2 --steps 4 --warmup 2 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:fine_ -s 2 -c 1 -o gpurun_out/full_c4_fine \
  python bench.py --workload C4 --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:coarse -s 2 -c 1 -o gpurun_out/full_c4_coarse \
  python bench.py --workload C4 --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
ls -la gpurun_out | tail -8
