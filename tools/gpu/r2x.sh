# the driver's N>1 code path (torch NCCL backend) with 2 ranks sharing the GPU (NCCL over loopback)
TAG=${1:-r2x}
mkdir -p gpurun_out
PYTHONUNBUFFERED=1 ACSR_BENCH_WATCHDOG=800 ACSR_SHARED_GPU_TEST=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --steps 10 --c4-scale 22 > gpurun_out/bench_tr2nccl_$TAG.json 2> gpurun_out/bench_tr2nccl_$TAG.err; tail -n 1 gpurun_out/bench_tr2nccl_$TAG.json | cut -c1-400; grep -v "UserWarning\|sparse_csr" gpurun_out/bench_tr2nccl_$TAG.err | tail -n 6
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref2_$TAG.json 2>/dev/null; tail -n 1 gpurun_out/bench_ref2_$TAG.json | cut -c1-300
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "property" 2>&1 | tail -n 2
