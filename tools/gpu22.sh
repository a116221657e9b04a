cd $GRAFT_REPO_ROOT
timeout 900 python bench.py > gpurun_out/bench9.json 2> gpurun_out/bench9.err
tail -2 gpurun_out/bench9.err; cat gpurun_out/bench9.json | head -c 3000; echo
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_ring_gemm -c 1 -o gpurun_out/tc4096v2b python tools/tc_sweep.py 4096 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_mlp_graph.csv python tools/step_profile.py mlp 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ring_gemm_small -s 4 -c 1 -o gpurun_out/small python tools/step_profile.py mlp 2 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
