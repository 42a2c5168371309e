#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
MG_DEBUG_FLAGS=${FLAGS:-0} timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:coarse_kernel -s 3 -c 1 -o gpurun_out/${NAME:-profx} \
  python bench.py --workload ${W:-C2} --steps 4 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${NAME:-profx}.log 2>&1
tail -2 gpurun_out/${NAME:-profx}.log
