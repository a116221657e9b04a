cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches64_cnn.csv python tools/step_profile.py cnn 2 > gpurun_out/ncu64.log 2>&1
tail -1 gpurun_out/ncu64.log
