#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
MG_UNIT_ORDER=2 timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi_item.py -m gpu -q -x 2>&1 | tail -1
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'])"; }
for rep in 1 2; do
for w in C2 C3 C5 QDS-LS; do
  for o in 1 2 0; do
    MG_UNIT_ORDER=$o timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 2>/dev/null | line "$w order=$o"
  done
done
done
for o in 1 2; do
  MG_UNIT_ORDER=$o timeout 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:coarse -s 3 -c 1 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | grep -E "dram__bytes|duration" | sed "s/^/order=$o /"
done
