#!/bin/bash
# GPU parity suite (optionally a subset: TESTS="tests/test_x.py -k y"); hard-killed on hang.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout -s KILL ${T:-900} python -m pytest ${TESTS:-tests} -m gpu -q -x ${PYARGS} 2>&1 | tail -${TAILN:-25}
