#!/bin/bash
# GPU-box job: per-phase globaltimer breakdown of tc_seg_kernel (TCSEG_TIMING build): MLP steps and
# stand-alone plain products (script given as $1, default tools/tcseg_timing.py).  Rebuilds normally at the end.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
PSML_NVCC_EXTRA=-DTCSEG_TIMING python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/tt_build.log 2>&1 || { tail -5 gpurun_out/tt_build.log; exit 1; }
for s in "$@"; do timeout 300 python $s; done
python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
