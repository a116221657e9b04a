cd $GRAFT_REPO_ROOT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cnn.csv python tools/step_profile.py cnn 2 > /dev/null 2>&1
wc -l gpurun_out/launches_cnn.csv
