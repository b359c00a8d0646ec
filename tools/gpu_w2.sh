TAG=${1:-w2}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf 2>&1 | tail -15 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json | cut -c1-900
timeout 900 python bench.py --steps 20 --warmup 3 --workload dynamic > gpurun_out/bench_dyn_$TAG.json 2>&1; tail -2 gpurun_out/bench_dyn_$TAG.json
timeout 900 python bench.py --steps 5 --warmup 3 --workload pagerank --scale 26 > gpurun_out/bench_pr26_$TAG.json 2>&1; tail -2 gpurun_out/bench_pr26_$TAG.json | cut -c1-900
timeout 600 python bench.py --steps 10 --warmup 3 --workload pagerank_dist --scale 24 > gpurun_out/bench_prd_$TAG.json 2>&1; tail -2 gpurun_out/bench_prd_$TAG.json | cut -c1-900
timeout 300 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"spmv_kernel|bin_|xc_|update_|pagerank_" --csv --log-file gpurun_out/launches_nc_$TAG.csv python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
