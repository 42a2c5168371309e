#!/bin/bash
# Fine kernel: hybrid K (TMA gather4) + V (cp.async) gathers (MG_FINE_HYB=1) vs cp.async only.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
MG_FINE_HYB=1 timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi_item.py -m gpu -q -x -k "fine or C4 or RBR or mixed or sm_split" 2>&1 | tail -2
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['roofline']['avg_launch_ms'],4), 'fine ms')"; }
for w in C4 F9-RBR F9-LBR DIL-LD; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w cp.async"
  MG_FINE_HYB=1 timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 200 2>/dev/null | line "$w hybrid"
done
