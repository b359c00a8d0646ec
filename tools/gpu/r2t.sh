TAG=${1:-r2t}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "dist or peer or acsr_comm or c_abi or exchange_layout or single_rank" 2>&1 | tail -n 3
PYTHONUNBUFFERED=1 ACSR_BENCH_WATCHDOG=800 ACSR_SHARED_GPU_TEST=1 ACSR_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 3 --master-addr 127.0.0.1 --master-port 29512 bench.py --no-cpu-baseline --steps 10 --c4-scale 20 > gpurun_out/bench_tr3_$TAG.json 2> gpurun_out/bench_tr3_$TAG.err; tail -n 1 gpurun_out/bench_tr3_$TAG.json | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(json.dumps(d['pagerank_dist'])[:1400])"
