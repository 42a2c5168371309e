#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'])"; }
for rep in 1 2; do
for w in C2 C3 C5; do
  for o in 1 0; do
    MG_UNIT_ORDER=$o timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 2>/dev/null | line "$w order=$o"
  done
done
done
