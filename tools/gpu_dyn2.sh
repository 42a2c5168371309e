#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['roofline']['avg_launch_ms'],4), 'fine ms')"; }
for w in C4 F9-RBR F9-LBR DIL-LD; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w auto"
  MG_FINE_DYN=0 timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w static"
done
timeout -s KILL 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
