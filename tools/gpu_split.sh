TAG=${1:-split}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "row_split" 2>&1 | tail -n 3
timeout 600 python bench.py --workload rmat20_split 2>gpurun_out/bench_split_$TAG.err | tail -n 1 > gpurun_out/bench_split_$TAG.jsonl
ACSR_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --workload rmat20_split --steps 10 2>>gpurun_out/bench_split_$TAG.err | tail -n 1 >> gpurun_out/bench_split_$TAG.jsonl
ACSR_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --workload pagerank_dist --scale 20 --steps 10 --exchange peer 2>>gpurun_out/bench_split_$TAG.err | tail -n 1 >> gpurun_out/bench_split_$TAG.jsonl
cut -c1-500 gpurun_out/bench_split_$TAG.jsonl; tail -n 5 gpurun_out/bench_split_$TAG.err
