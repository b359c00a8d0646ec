# usage: bash tools/gpu_wide.sh <tag>
TAG=${1:-w}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf 2>&1 | tail -15 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
timeout 300 python bench.py --steps 20 --warmup 5 --workload rmat20_f32 --no-cpu-baseline > gpurun_out/bench_f32_$TAG.json 2>&1; tail -1 gpurun_out/bench_f32_$TAG.json | cut -c1-700
timeout 300 python bench.py --steps 20 --warmup 5 --workload webgoogle --no-cpu-baseline > gpurun_out/bench_wg_$TAG.json 2>&1; tail -1 gpurun_out/bench_wg_$TAG.json | cut -c1-700
timeout 300 python bench.py --steps 20 --warmup 5 --workload livejournal --no-cpu-baseline > gpurun_out/bench_lj_$TAG.json 2>&1; tail -1 gpurun_out/bench_lj_$TAG.json | cut -c1-700
timeout 600 python bench.py --steps 10 --warmup 3 --workload pagerank --scale 22 > gpurun_out/bench_pr22_$TAG.json 2>&1; tail -1 gpurun_out/bench_pr22_$TAG.json
timeout 900 python bench.py --steps 10 --warmup 3 --workload pagerank --scale 26 > gpurun_out/bench_pr26_$TAG.json 2>&1; tail -2 gpurun_out/bench_pr26_$TAG.json
timeout 900 python bench.py --steps 20 --warmup 3 --workload dynamic > gpurun_out/bench_dyn_$TAG.json 2>&1; tail -2 gpurun_out/bench_dyn_$TAG.json
timeout 300 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"spmv_kernel|bin_|xc_|update_|pagerank_" --csv --log-file gpurun_out/launches_nc_$TAG.csv python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
