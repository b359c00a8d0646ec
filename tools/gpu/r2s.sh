TAG=${1:-r2s}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
PYTHONUNBUFFERED=1 ACSR_BENCH_WATCHDOG=800 ACSR_SHARED_GPU_TEST=1 ACSR_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 3 --master-addr 127.0.0.1 --master-port 29512 bench.py --no-cpu-baseline --steps 10 --c4-scale 20 > gpurun_out/bench_tr3_$TAG.json 2> gpurun_out/bench_tr3_$TAG.err; tail -n 1 gpurun_out/bench_tr3_$TAG.json | cut -c1-300; grep -v "UserWarning\|sparse_csr" gpurun_out/bench_tr3_$TAG.err | tail -n 5
