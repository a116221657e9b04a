cd $GRAFT_REPO_ROOT
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ring_gemm_small -s 2 -c 3 -o gpurun_out/small35 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/ncu35.log 2>&1
tail -2 gpurun_out/ncu35.log
