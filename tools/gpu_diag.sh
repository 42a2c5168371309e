#!/bin/bash
# Coarse-kernel diagnostics: per-tile timelines (MG_TIMELINE variants: normal, no exp, skeleton) and
# the bench ms of the MG_DBG skeleton builds on C2.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for v in ${TLV:-timeline tl1 tl7}; do
  python -m paper_conf_iiswc_lica22_b200.build --variant $v > /dev/null || echo "build $v failed"
  MG_LIB_VARIANT=$v timeout -s KILL 120 python tools/timeline_pp.py ${W:-C2} > gpurun_out/diag_tl_$v.txt 2>&1
done
for v in ${DBGV:-dbg1 dbg2 dbg7}; do
  python -m paper_conf_iiswc_lica22_b200.build --variant $v > /dev/null || echo "build $v failed"
done
VARIANTS="${DBGV:-dbg1 dbg2 dbg7}" STEPS=300 bash tools/ab_variants.sh > gpurun_out/diag_ab.txt 2>&1
