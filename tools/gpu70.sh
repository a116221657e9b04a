cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_mlp.json 2>&1 | tail -80
PSML_DEAL_CTAS=0 timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_mlp0.json 2>&1 | grep -E "mean step|busy"
