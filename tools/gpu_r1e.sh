TAG=${1:-r1e}
mkdir -p gpurun_out
timeout 300 ./tools/bin/gather_bench big > gpurun_out/gather_bench_big.jsonl 2>&1; head -8 gpurun_out/gather_bench_big.jsonl
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -k "boundary or empty or update or edge_sizes or unaligned or grow or closed_forms" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1; tail -8 gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or bins_bitwise_rmat" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1; tail -8 gpurun_out/sanitizer_racecheck_$TAG.txt
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or integer_bitwise_boundary" > gpurun_out/sanitizer_synccheck_$TAG.txt 2>&1; tail -8 gpurun_out/sanitizer_synccheck_$TAG.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_|update_|pagerank_|xc_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_spmv_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"bin_" -s 3 -c 3 -o gpurun_out/prof_bin_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bin_$TAG.log 2>&1
ls gpurun_out | grep $TAG
