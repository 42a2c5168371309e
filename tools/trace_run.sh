# Diagnostics: MG_TRACE build -> per-phase cycle breakdown of the coarse kernel's roles (wet and
# with each MG_DEBUG_FLAGS value in TRACE_FLAGS), then the normal build is restored.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
MG_TRACE=1 python -m paper_conf_iiswc_lica22_b200.build > /dev/null
W=${WORKLOAD:-C2}
timeout -s KILL 120 python tools/trace_coarse.py $W > gpurun_out/trace_$W.txt 2>&1
for f in ${TRACE_FLAGS:-7}; do
  MG_DEBUG_FLAGS=$f timeout -s KILL 120 python tools/trace_coarse.py $W > gpurun_out/trace_${W}_f$f.txt 2>&1
done
python -m paper_conf_iiswc_lica22_b200.build > /dev/null
