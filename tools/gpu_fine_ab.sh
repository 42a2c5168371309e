#!/bin/bash
# Fine-kernel check: its parity tests, C4 / F9-RBR bench lines, and instruction / time counters of one launch.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi_item.py -m gpu -q -x -k "fine or C4 or RBR or mixed" 2>&1 | tail -3
for w in C4 F9-RBR F9-LBR; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps ${STEPS:-100} 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'], d['roofline'].get('l2'))"
done
timeout 300 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,lts__t_sectors.sum --clock-control none -k regex:fine -s 2 -c 1 python bench.py --workload C4 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | grep -E "fine|duration|inst_executed|issue_active|sectors" | head -8
