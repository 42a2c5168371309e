#!/bin/bash
# ncu warp-state / source-level stall capture of the C2 coarse kernel (one launch).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:coarse -s 4 -c 1 -o gpurun_out/stall_c2 -f python bench.py --steps 6 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/stall_c2.log 2>&1
ncu -i gpurun_out/stall_c2.ncu-rep --page details --csv > gpurun_out/stall_c2_details.csv 2>&1
ncu -i gpurun_out/stall_c2.ncu-rep --page source --csv --print-source sass > gpurun_out/stall_c2_source.csv 2>&1
ls -la gpurun_out/stall_c2*
