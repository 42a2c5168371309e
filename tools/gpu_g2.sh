cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
TESTS="tests/test_gpu_staged.py" bash tools/gpu_tests.sh
timeout -s KILL 300 python bench.py --steps 500 > gpurun_out/b2_C2.json 2>gpurun_out/b2_C2.err; tail -2 gpurun_out/b2_C2.err
timeout -s KILL 300 python bench.py --workload C5 --no-cpu-baseline --steps 200 > gpurun_out/b2_C5.json 2>gpurun_out/b2_C5.err; tail -2 gpurun_out/b2_C5.err
timeout -s KILL 300 python bench.py --workload C4 --no-cpu-baseline --steps 100 > gpurun_out/b2_C4.json 2>gpurun_out/b2_C4.err; tail -2 gpurun_out/b2_C4.err
timeout -s KILL 300 python bench.py --workload C3 --no-cpu-baseline --steps 300 --ablation > gpurun_out/b2_C3.json 2>gpurun_out/b2_C3.err; tail -2 gpurun_out/b2_C3.err
