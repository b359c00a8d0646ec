# round-2: full GPU suite + capi + bench N=1, torchrun N=1, torchrun N=2 on one GPU (test knob)
TAG=${1:-r2c}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x -rf 2>&1 | tail -n 15 > gpurun_out/pytest_gpu_$TAG.txt; tail -n 6 gpurun_out/pytest_gpu_$TAG.txt
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-300; tail -n 3 gpurun_out/bench_$TAG.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --no-cpu-baseline > gpurun_out/bench_tr1_$TAG.json 2> gpurun_out/bench_tr1_$TAG.err; tail -n 1 gpurun_out/bench_tr1_$TAG.json | cut -c1-300; tail -n 3 gpurun_out/bench_tr1_$TAG.err
NCCL_DEBUG=INFO ACSR_SHARED_GPU_TEST=1 ACSR_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --no-cpu-baseline --steps 10 > gpurun_out/bench_tr2_$TAG.json 2> gpurun_out/bench_tr2_$TAG.err; tail -n 1 gpurun_out/bench_tr2_$TAG.json | cut -c1-300; grep -v "NCCL INFO" gpurun_out/bench_tr2_$TAG.err | tail -n 5
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2>&1; tail -n 1 gpurun_out/bench_ref_$TAG.json | cut -c1-300
