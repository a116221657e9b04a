cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_NVCC_EXTRA=-DTCSEG_TIMING python -m paper_conf_icpp_chenzzzz020_b200.build --force 2>&1 | grep -i error
stdbuf -o0 -e0 timeout 120 python tools/step_profile.py mlp 3 > gpurun_out/t50.txt 2>&1
grep -c tcseg gpurun_out/t50.txt
grep tcseg gpurun_out/t50.txt | tail -24
