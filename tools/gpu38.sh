cd $GRAFT_REPO_ROOT
timeout 120 python tools/gemm_lat.py 1
PSML_SIMT=small timeout 120 python tools/gemm_lat.py 1
timeout 120 python tools/gemm_lat.py 2
