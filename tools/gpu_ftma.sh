cd "${GRAFT_REPO_ROOT:-/root/repo}"
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi_item.py tests/test_gpu_block64.py -m gpu -q -x 2>&1 | tail -3
for tma in 1 0; do
  for w in C4 F9-RBR F9-LBR; do
    MG_FINE_TMA=$tma timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('tma=$tma $w', round(d['ms_per_step'],4), round(d['roofline']['avg_launch_ms'],4))"
  done
done
