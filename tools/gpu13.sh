cd $GRAFT_REPO_ROOT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_graph.csv python tools/step_profile.py mlp 3 > gpurun_out/ncu13.log 2>&1
tail -2 gpurun_out/ncu13.log; wc -l gpurun_out/launches_graph.csv
