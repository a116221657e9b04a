cd $GRAFT_REPO_ROOT
for d in 0 1 2 3; do echo "debug=$d"; PSML_TC_DEBUG=$d timeout 300 python tools/tc_sweep.py 4096,8192 2>&1 | grep '"backend": 2' | grep '"l": 64'; done
