cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
# launch list of the bench command (first launches: warm-up eager steps, then graph steps)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches46_bench.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/ncu46a.log 2>&1
tail -2 gpurun_out/ncu46a.log
# launch list of pure pipelined graph steps
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches46_graph.csv python tools/step_profile.py mlp 4 > gpurun_out/ncu46b.log 2>&1
tail -2 gpurun_out/ncu46b.log
# full capture of the top kernels in one graph step
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"seg_gemm|msb_chain|deal_prg|gemm_small|open_list|had_fused|update_all" -s 30 -c 12 -o gpurun_out/full46 python tools/step_profile.py mlp 3 > gpurun_out/ncu46c.log 2>&1
tail -2 gpurun_out/ncu46c.log
ls -la gpurun_out
