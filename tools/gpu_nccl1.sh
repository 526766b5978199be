# the NCCL data path (weight broadcast, per-step logits all-gather) on one B200:
# a 1-rank NCCL group, direct and under torchrun
cd $GRAFT_REPO_ROOT
NCCL_DEBUG=INFO timeout 600 python bench.py --nccl --net vgg16 --global-batch 1024 --no-sweep --no-extra --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/nccl1_direct.json 2> gpurun_out/nccl1_direct.err; echo direct=$?
NCCL_DEBUG=INFO timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 1 --nccl --no-sweep --no-extra --no-cpu-baseline --steps 20 > gpurun_out/nccl1_torchrun.json 2> gpurun_out/nccl1_torchrun.err; echo torchrun=$?
grep -h "NCCL INFO" gpurun_out/nccl1_direct.err | head -5
for f in gpurun_out/nccl1_direct.json gpurun_out/nccl1_torchrun.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print(d['config'].get('workload'), d['value'], d['nccl'], d['weights_broadcast_ms'], d.get('logits_sha256','')[:16], d['e2e']['api'])"; done
