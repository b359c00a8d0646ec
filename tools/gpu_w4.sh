TAG=${1:-w4}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf 2>&1 | tail -8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 900 python bench.py --workload dynamic_mixed > gpurun_out/bench_dynmix_$TAG.json 2>&1; tail -1 gpurun_out/bench_dynmix_$TAG.json
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 2 --relabel > gpurun_out/bench_pr26r_$TAG.json 2>&1; tail -1 gpurun_out/bench_pr26r_$TAG.json
timeout 900 python bench.py --workload pagerank --scale 22 --steps 10 --warmup 3 --relabel > gpurun_out/bench_pr22r_$TAG.json 2>&1; tail -1 gpurun_out/bench_pr22r_$TAG.json
