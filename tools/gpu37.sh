cd $GRAFT_REPO_ROOT
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ring_gemm_cl -s 3 -c 2 -o gpurun_out/cl37 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/ncu37.log 2>&1
tail -2 gpurun_out/ncu37.log
