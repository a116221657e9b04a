cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_NVCC_EXTRA=-DTCSEG_TIMING python -m paper_conf_icpp_chenzzzz020_b200.build --force 2>&1 | grep -i error
for mm in 0 1 8; do
PSML_TCSEG_MMAS=$mm stdbuf -o0 -e0 timeout 120 python tools/step_profile.py mlp 3 > gpurun_out/t54_$mm.txt 2>&1
echo "MMAS=$mm"; grep "grid 4 .*nblk 4" gpurun_out/t54_$mm.txt | tail -2; grep "grid 28 " gpurun_out/t54_$mm.txt | tail -1
done
