cd $GRAFT_REPO_ROOT
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -5 gpurun_out/bench1.err
cat gpurun_out/bench1.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches1.csv python bench.py --steps 2 --warmup 1 --no-ring-gemm --no-cpu-baseline > /dev/null 2>&1
wc -l gpurun_out/launches1.csv
