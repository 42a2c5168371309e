#!/bin/bash
# compute-sanitizer racecheck / synccheck / memcheck over tools/sanitize_run.py (one GPU, bounded).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for tool in ${TOOLS:-racecheck synccheck memcheck}; do
  echo "=== $tool"
  timeout -s KILL ${T:-900} compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py 2>&1 | tail -25
done
