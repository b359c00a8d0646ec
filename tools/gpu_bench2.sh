TAG=${1:-b2}
mkdir -p gpurun_out
ACSR_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29535 bench.py --gpus 2 --steps 10 --warmup 3 2>gpurun_out/bench2_$TAG.err | tail -n 1 > gpurun_out/bench2_$TAG.jsonl
ACSR_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29536 bench.py --impl reference --gpus 2 --steps 2 --warmup 3 2>>gpurun_out/bench2_$TAG.err | tail -n 1 >> gpurun_out/bench2_$TAG.jsonl
cut -c1-300 gpurun_out/bench2_$TAG.jsonl; python -c "
import json
l=json.loads(open('gpurun_out/bench2_$TAG.jsonl').readline()); print(l['e2e'], 'cpu_baseline' in l, l['n_gpus'], l['value'])"
tail -n 3 gpurun_out/bench2_$TAG.err
