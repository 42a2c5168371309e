#!/bin/bash
# SM-split mode (plan concurrency 3): its parity tests, then C4 / F9-RBR / DIL-LD bench lines for
# serial, two-stream concurrent and SM split (auto share, and MG_SPLIT_CTAS overrides).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi_item.py -m gpu -q -x -k "sm_split or 3" 2>&1 | tail -3
line() { python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), 'ms', round(d['value'],1), d['unit'])"; }
for w in ${W:-C4 F9-RBR DIL-LD}; do
  for c in 1 2 3; do
    timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps ${STEPS:-100} --concurrency $c 2>/dev/null | line "$w conc=$c" || echo "$w conc=$c FAILED"
  done
  for n in ${NS:-8 16 32 64}; do
    MG_SPLIT_CTAS=$n timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps ${STEPS:-100} --concurrency 3 2>/dev/null | line "$w split=$n" || echo "$w split=$n FAILED"
  done
done
