#!/bin/bash
# GPU parity (coarse-heavy subset) + bench lines of C2/C3/C4 (no profiler); hard-killed on hang.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_gpu_multi_item.py tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -4
for w in ${WORKLOADS:-C2 C3 C4}; do
  timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  python -c "
import json;d=json.load(open('gpurun_out/bench_$w.json'))
r=d['roofline']
print('$w', 'TFLOP/s', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'med', round(d['fwd_ms']['median'],4), 'frac', round(r['frac'],4), 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
" 2>/dev/null || { echo "$w FAILED/HUNG"; tail -3 gpurun_out/bench_$w.err; }
done
