TAG=${1:-w3}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf 2>&1 | tail -15 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
timeout 300 python bench.py --workload hits --warmup 3 > gpurun_out/bench_hits_$TAG.json 2>&1; tail -1 gpurun_out/bench_hits_$TAG.json
timeout 300 python bench.py --workload rwr --warmup 3 > gpurun_out/bench_rwr_$TAG.json 2>&1; tail -1 gpurun_out/bench_rwr_$TAG.json
timeout 600 python bench.py --workload pagerank_dist --scale 24 --steps 10 --warmup 3 > gpurun_out/bench_prd_$TAG.json 2>&1; tail -1 gpurun_out/bench_prd_$TAG.json
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>&1; tail -1 gpurun_out/bench_ref_$TAG.json
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
