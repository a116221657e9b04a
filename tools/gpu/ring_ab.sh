#!/bin/bash
# GPU-box job: ring GEMM timings for compile-time variants.  Usage: ring_ab.sh "<flags A>" "<flags B>" ...
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for flags in "$@"; do
  PSML_NVCC_EXTRA="$flags" python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/ring_ab_build.log 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== [$flags]"; timeout 300 python tools/ring_sweep_quick.py ${RING_NS:-512 1024 2048 4096}
done
