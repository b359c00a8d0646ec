# session-3 evidence pass on the final code: tests, smoke, bench lines, ncu, sanitizers
TAG=${1:-r1q}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 6 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-300
: > gpurun_out/bench_lines_$TAG.jsonl
for wl in rmat20_f32 webgoogle livejournal; do timeout 300 python bench.py --workload $wl --no-cpu-baseline 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl; done
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 --relabel 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload pagerank_dist --scale 26 --steps 5 --warmup 3 --exchange peer 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload dynamic 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 900 python bench.py --workload dynamic_mixed 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --workload hits 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --workload rwr 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --workload rmat20_split 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 2>/dev/null | tail -n 1 >> gpurun_out/bench_lines_$TAG.jsonl
cut -c1-160 gpurun_out/bench_lines_$TAG.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_|update_|pagerank_|xc_|hits_|peer_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"bin_" -s 9 -c 3 -o gpurun_out/prof_bin_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_parity.py -q -x -k "boundary or empty or update or edge_sizes or unaligned or grow or closed_forms or long_row or hits or rwr or peer_exchange_single" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or bins_bitwise_rmat or long_row or window_rows" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_racecheck_$TAG.txt
ls gpurun_out | grep $TAG
