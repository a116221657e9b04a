#!/bin/bash
# GPU-box job: the gpu test suite (optionally filtered) + smoke.  Usage: tests.sh [pytest -k expr]
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$1" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q -k "$1" 2>&1 | tail -40
else
  timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -40
fi
