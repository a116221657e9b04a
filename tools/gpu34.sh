cd $GRAFT_REPO_ROOT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launch34.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/b34.log 2>&1
tail -2 gpurun_out/b34.log
timeout 300 ncu --set full --clock-control none --import-source on -k regex:deal_ -c 2 -o gpurun_out/deal34 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/ncu34.log 2>&1
tail -2 gpurun_out/ncu34.log
