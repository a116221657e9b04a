cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r01c_launches_bench.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/ncu58a.log 2>&1
tail -1 gpurun_out/ncu58a.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01c_launches_graph.csv python tools/step_profile.py mlp 4 > gpurun_out/ncu58b.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"seg_gemm|tc_seg|msb_chain|deal_prg|ring_gemm_cl" -s 20 -c 10 -o gpurun_out/r01c_full python tools/step_profile.py mlp 3 > gpurun_out/ncu58c.log 2>&1
tail -1 gpurun_out/ncu58c.log
