cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
for w in C2 C3 C4; do timeout -s KILL 120 python bench.py --workload $w --no-cpu-baseline --steps 300 > gpurun_out/b0_$w.json 2>gpurun_out/b0_$w.err; done
MG_LIB_VARIANT=timeline timeout -s KILL 120 python tools/timeline_pp.py C2 > gpurun_out/tl0_c2.txt 2>&1
MG_LIB_VARIANT=timeline timeout -s KILL 120 python tools/timeline_pp.py C2 --dump 5 > gpurun_out/tl0_c2_d5.txt 2>&1
