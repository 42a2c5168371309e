#!/bin/bash
# Unit order A/B: item-major in groups of (b,h) units with items by decreasing tile count (default,
# MG_UNIT_GROUP overrides the group size) vs (b,h)-major (MG_UNIT_ORDER=0).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
timeout -s KILL 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'])"; }
for w in C2 C3 C5 C4 QDS-LS; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 2>/dev/null | line "$w group96"
  MG_UNIT_ORDER=0 timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 2>/dev/null | line "$w bh-major"
done
for g in 24 48 192; do
  for w in C2 C5; do
    MG_UNIT_GROUP=$g timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 2>/dev/null | line "$w group$g"
  done
done
