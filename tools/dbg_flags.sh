# Diagnostics: C2 bench time with each MG_DEBUG_FLAGS value in FLAGS (results are garbage).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for f in ${FLAGS:-0 1 64 65}; do
  MG_DEBUG_FLAGS=$f timeout -s KILL 60 python bench.py --workload ${W:-C2} --no-cpu-baseline --steps 200 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('flags $f', round(d['ms_per_step'],4))"
done
