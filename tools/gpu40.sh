cd $GRAFT_REPO_ROOT/tools/micro
timeout 300 ncu --set full --cache-control none --clock-control none --import-source on -k regex:ring_gemm_cl -c 6 -o ../../gpurun_out/micro40 ./gemm_micro prof > ../../gpurun_out/ncu40.log 2>&1
tail -2 ../../gpurun_out/ncu40.log
