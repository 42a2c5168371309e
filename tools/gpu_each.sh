cd "${GRAFT_REPO_ROOT:-/root/repo}"
for t in $(python -m pytest tests/test_gpu_d128.py -m gpu --collect-only -q 2>/dev/null | grep "::"); do
  r=$(timeout -s KILL 60 python -m pytest "$t" -m gpu -q -x 2>&1 | tail -1)
  echo "$t => $r"
done
