#!/bin/bash
# ncu full capture of one launch of a kernel: tools/gpu_prof.sh <workload> <kernel-regex> <name>
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
W=${1:-C2}; K=${2:-coarse_kernel}; N=${3:-prof}
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 -o gpurun_out/$N \
  python bench.py --workload $W --steps 4 --warmup 2 --no-cpu-baseline --e2e-steps 1 > gpurun_out/$N.log 2>&1
tail -3 gpurun_out/$N.log
