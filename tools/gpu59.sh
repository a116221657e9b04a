cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_DIST_BACKEND=gloo PSML_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --deployment split --steps 5 --warmup 3 > gpurun_out/b59s.json 2> gpurun_out/b59s.err
tail -3 gpurun_out/b59s.err; cat gpurun_out/b59s.json
timeout 900 python bench.py > gpurun_out/b59.json 2> gpurun_out/b59.err
tail -2 gpurun_out/b59.err
python -c "
import json; d=json.load(open('gpurun_out/b59.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print(d['roofline']); print(d['beaver_matmul_cfg1']); print(d['cpu_baseline']); print([ (g['n'],g['l'],round(g['ms'],3),round(g['useful_limb_tops'])) for g in d['ring_gemm']])"
