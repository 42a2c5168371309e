#!/bin/bash
# Fine kernel: static grid-stride rows vs dynamically claimed row chunks (MG_FINE_DYN=1), serial mode.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['roofline']['avg_launch_ms'],4), 'fine ms')"; }
for rep in 1 2; do
for w in C4 F9-RBR F9-LBR DIL-LD; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w static"
  MG_FINE_DYN=1 timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w dyn"
done
done
MG_FINE_DYN=1 timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "fine or C4 or RBR" 2>&1 | tail -2
