#!/bin/bash
# A/B: bench ms of the default library and of each MG_LIB_VARIANT in VARIANTS (workload W).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for v in default ${VARIANTS}; do
  if [ "$v" = default ]; then unset MG_LIB_VARIANT; else export MG_LIB_VARIANT=$v; fi
  for w in ${W:-C2}; do
    timeout -s KILL 90 python bench.py --workload $w --no-cpu-baseline --steps ${STEPS:-300} 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v $w', round(d['ms_per_step'],4), 'TFLOP/s', round(d['value'],1))" || echo "$v $w FAILED"
  done
done
# extra: default library with each MG_DEBUG_FLAGS value in XFLAGS
unset MG_LIB_VARIANT
for f in ${XFLAGS}; do
  for w in ${W:-C2}; do
    MG_DEBUG_FLAGS=$f timeout -s KILL 90 python bench.py --workload $w --no-cpu-baseline --steps ${STEPS:-300} 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('flags $f $w', round(d['ms_per_step'],4), 'TFLOP/s', round(d['value'],1))" || echo "flags $f $w FAILED"
  done
done
