#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py, default and with the fine kernel's dynamic rows forced.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for dyn in "" 1; do
  for tool in racecheck synccheck memcheck; do
    echo "=== $tool MG_FINE_DYN=$dyn"
    MG_FINE_DYN=$dyn timeout -s KILL 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py 2>&1 | tail -14
  done
done
