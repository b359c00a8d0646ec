# round-2 evidence pass: GPU suite, smoke, default bench (N=1, torchrun N=1, 2 ranks on one GPU), every bench line
TAG=${1:-r2m}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 6 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-200
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --no-cpu-baseline > gpurun_out/bench_tr1_$TAG.json 2>/dev/null; tail -n 1 gpurun_out/bench_tr1_$TAG.json | cut -c1-200
PYTHONUNBUFFERED=1 ACSR_BENCH_WATCHDOG=800 ACSR_SHARED_GPU_TEST=1 ACSR_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --no-cpu-baseline --steps 10 --c4-scale 22 > gpurun_out/bench_tr2_$TAG.json 2> gpurun_out/bench_tr2_$TAG.err; tail -n 1 gpurun_out/bench_tr2_$TAG.json | cut -c1-200
: > gpurun_out/bench_lines_$TAG.jsonl
for wl in rmat20_f32 webgoogle livejournal; do timeout 300 python bench.py --workload $wl --no-cpu-baseline --no-c4 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl; done
timeout 900 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 --relabel 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload dynamic 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload dynamic_mixed 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --workload hits 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --workload rwr 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
cut -c1-160 gpurun_out/bench_lines_$TAG.jsonl
