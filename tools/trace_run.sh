# Diagnostics: MG_TIMELINE build -> per-item boundary timeline; MG_TRACE build -> per-phase
# cycle breakdown (register heavy: perturbs the schedule); then the normal build is restored.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
MG_TIMELINE=1 python -m paper_conf_iiswc_lica22_b200.build > /dev/null
for W in ${WORKLOADS:-C2}; do
  timeout -s KILL 120 python tools/timeline_coarse.py $W > gpurun_out/timeline_$W.txt 2>&1
done
if [ -n "$PHASES" ]; then
  MG_TRACE=1 python -m paper_conf_iiswc_lica22_b200.build > /dev/null
  for W in ${WORKLOADS:-C2}; do
    timeout -s KILL 120 python tools/trace_coarse.py $W > gpurun_out/trace_$W.txt 2>&1
  done
fi
python -m paper_conf_iiswc_lica22_b200.build > /dev/null
