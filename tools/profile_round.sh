#!/bin/bash
# Round profile capture (one GPU), in two parts so that each call's gpurun_out stays under 64 MiB:
#   bash tools/profile_round.sh 1   launch lists (C2, C3, C4, C2 at d=128) + full captures C2 / C3 coarse
#   bash tools/profile_round.sh 2   full captures C4 fine, C4 coarse, C2 coarse at d=128
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
cap() {  # name regex workload-args...
  local name=$1 rx=$2; shift 2
  timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:$rx -s 3 -c 1 -o gpurun_out/$name \
    python bench.py "$@" --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
}
if [ "${1:-1}" = 1 ]; then
  for W in C2 C3 C4; do
    timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_$W.csv python bench.py --workload $W --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
  done
  timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_C2-d128.csv python bench.py --workload C2 --head-dim 128 --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
  cap full_c2_coarse coarse --workload C2
  cap full_c3_coarse coarse --workload C3
else
  cap full_c4_fine fine_ --workload C4
  cap full_c4_coarse coarse --workload C4
  cap full_c2d128_coarse coarse --workload C2 --head-dim 128
fi
ls -la gpurun_out | tail -12
