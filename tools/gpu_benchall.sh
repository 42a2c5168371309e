#!/bin/bash
# All bench lines of the round (no profiler): default C2 (with the CPU baseline), C3, C4, C5 at N=1,
# C2 at d=128 / b=64, the extra workloads, the staged ablation; one JSON line each in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
run() { local tag=$1; shift; timeout -s KILL 300 python bench.py "$@" > gpurun_out/ball_$tag.json 2> gpurun_out/ball_$tag.err || echo "$tag FAILED"; }
run C2 --steps 1000
run C2ref --impl reference --steps 5 --warmup 3
run C3 --workload C3 --no-cpu-baseline --steps 500 --ablation
run C4 --workload C4 --no-cpu-baseline --steps 100
run C5 --workload C5 --no-cpu-baseline --steps 200
run C2d128 --head-dim 128 --no-cpu-baseline --steps 500
run C2b64 --block 64 --no-cpu-baseline --steps 500
run C2abl --no-cpu-baseline --steps 300 --ablation
for w in QDS-LS F9-LS F9-LSG F9-LBR F9-RBR DIL-LD; do run $w --workload $w --no-cpu-baseline --steps 300; done
python - <<'PY'
import json, glob, os
for f in sorted(glob.glob("gpurun_out/ball_*.json")):
    try:
        d = json.load(open(f))
    except Exception as e:
        print(os.path.basename(f), "ERR", e); continue
    r = d.get("roofline", {})
    print(os.path.basename(f)[5:-5], round(d["ms_per_step"], 4), "ms", round(d["value"], 1), d["unit"], "frac", round(r.get("frac", 0), 3),
          "l2", round(r.get("l2", {}).get("frac", 0), 3), "e2e", round(d.get("e2e", {}).get("value", 0), 2), d.get("clocks", {}).get("sm_mhz"), d.get("clocks", {}).get("reasons"))
PY
