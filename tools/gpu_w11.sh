TAG=${1:-w11}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf 2>&1 | tail -8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 900 python bench.py --workload dynamic > gpurun_out/bench_dyn_$TAG.json 2>&1; tail -1 gpurun_out/bench_dyn_$TAG.json
timeout 300 python bench.py --workload rwr --warmup 3 > gpurun_out/bench_rwr_$TAG.json 2>&1; tail -1 gpurun_out/bench_rwr_$TAG.json
timeout 600 python bench.py --steps 10 --warmup 3 --workload pagerank --scale 22 > gpurun_out/bench_pr22_$TAG.json 2>&1; tail -1 gpurun_out/bench_pr22_$TAG.json | cut -c1-600
