#!/bin/bash
# Parity tests + bench lines (no profiler). Every step is hard-killed on hang.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout -s KILL 240 python -m pytest tests -m gpu -q -x 2>&1 | tail -15
for w in ${WORKLOADS:-C2 C3 C4}; do
  timeout -s KILL 90 python bench.py --workload $w --no-cpu-baseline --steps 300 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  python -c "
import json;d=json.load(open('gpurun_out/bench_$w.json'))
r=d['roofline']
print('$w', 'TFLOP/s', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'kernel', r['kernel'][:14], 'frac', round(r['frac'],4), 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
" 2>/dev/null || echo "$w FAILED/HUNG"
done
