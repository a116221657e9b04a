#!/bin/bash
# GPU-box job: the default bench line, its ncu launch list, and ncu --set full captures of the
# step's top kernels and of the config-5 ring GEMM.  Usage: bench.sh TAG   (outputs gpurun_out/TAG_*)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
T=${1:-r02}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
echo "bench rc=$?"; tail -c 1500 gpurun_out/${T}_bench.json; tail -3 gpurun_out/${T}_bench.err
if [ "$2" != "nocu" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${T}_launches.csv \
  python bench.py --steps 20 --warmup 3 --no-ring-gemm --no-cpu-baseline --no-classes --no-secondary > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"seg_gemm|tc_seg|msb_chain|had_fused|open_list|deal_prg" \
  -s 400 -c 12 -o gpurun_out/${T}_full python bench.py --steps 20 --warmup 3 --no-ring-gemm --no-cpu-baseline --no-classes --no-secondary > /dev/null 2>&1; echo "ncu full rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"tc_ring|tc_finalize|split" -c 6 \
  -o gpurun_out/${T}_ring4096 python tools/ring_gemm_once.py 4096 64 1 > /dev/null 2>&1; echo "ncu ring rc=$?"
fi
