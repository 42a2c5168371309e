#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for f in ${FLAGS:-0 1}; do
  MG_DEBUG_FLAGS=$f timeout -s KILL 90 python bench.py --no-cpu-baseline --steps 200 --workload ${W:-C2} > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));print('flags', $f, round(d['ms_per_step'],4), round(d['roofline']['avg_launch_ms'],4))"
done
