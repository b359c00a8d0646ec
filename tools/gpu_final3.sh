TAG=${1:-r1m}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 4 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-200
: > gpurun_out/bench_lines_$TAG.jsonl
for wl in rmat20_f32 webgoogle livejournal rmat20_split hits rwr dynamic dynamic_mixed; do timeout 600 python bench.py --workload $wl --no-cpu-baseline 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl; done
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 --relabel 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload pagerank_dist --scale 26 --steps 5 --warmup 3 --exchange peer 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
cut -c1-150 gpurun_out/bench_lines_$TAG.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_parity.py -q -x -k "update or epoch or long_row or prefetch_views or boundary or empty" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1; tail -n 2 gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -k "long_row_cta or epoch" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1; tail -n 2 gpurun_out/sanitizer_racecheck_$TAG.txt
