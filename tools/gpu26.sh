cd $GRAFT_REPO_ROOT
timeout 900 python tools/cnn_drift.py 2>&1 | tail -8
