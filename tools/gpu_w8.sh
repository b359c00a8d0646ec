TAG=${1:-w8}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf 2>&1 | tail -8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 900 python bench.py --workload dynamic_mixed > gpurun_out/bench_dynmix_$TAG.json 2>&1; tail -1 gpurun_out/bench_dynmix_$TAG.json
timeout 900 python bench.py --workload dynamic > gpurun_out/bench_dyn_$TAG.json 2>&1; tail -1 gpurun_out/bench_dyn_$TAG.json
