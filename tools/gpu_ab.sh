#!/bin/bash
# Parity subset + A/B of library variants: TESTS (pytest selection, optional), VARIANTS (build.py
# variant names, built on the box), W (workloads), STEPS.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
if [ -n "$TESTS" ]; then
  timeout -s KILL ${T:-600} python -m pytest $TESTS -m gpu -q -x 2>&1 | tail -${TAILN:-15}
fi
for v in ${VARIANTS}; do python -m paper_conf_iiswc_lica22_b200.build --variant $v > /dev/null || echo "build $v failed"; done
bash tools/ab_variants.sh
