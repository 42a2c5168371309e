#!/bin/bash
# Dense-row items split into column chunks (forced, --dense-chunk N) vs the default rule, C2 / C3 / F9-LSG.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'])"; }
for w in C2 C3 F9-LSG; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 400 2>/dev/null | line "$w default"
  for dc in 4 8 16; do
    timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 400 --dense-chunk $dc 2>/dev/null | line "$w chunk=$dc"
  done
done
