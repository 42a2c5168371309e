#!/bin/bash
# ncu warp-state / source-level stall capture of one kernel launch: K (kernel regex, default coarse),
# W (workload, default C2), TAG (output name).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
K=${K:-coarse}; W=${W:-C2}; TAG=${TAG:-stall_c2}
timeout 600 ncu --set full --import-source on --clock-control none -k regex:$K -s 2 -c 1 -o gpurun_out/$TAG -f python bench.py --workload $W --steps 4 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/$TAG.log 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>&1
ncu -i gpurun_out/$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_source.csv 2>&1
ls -la gpurun_out/$TAG*
