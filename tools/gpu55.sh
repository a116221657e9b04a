cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_NVCC_EXTRA=-DTCSEG_TIMING python -m paper_conf_icpp_chenzzzz020_b200.build --force 2>&1 | grep -i error
stdbuf -o0 -e0 timeout 120 python tools/step_profile.py mlp 2 > gpurun_out/t55.txt 2>&1
grep -A0 "blk i=\|grid 4 blk 0 z 0" gpurun_out/t55.txt | tail -16
