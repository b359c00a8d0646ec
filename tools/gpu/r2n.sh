# round-2 profiler + sanitizer evidence on the final code
TAG=${1:-r2n}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_|update_|pagerank_|xc_|hits_|peer_|relabel|comm" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-c4 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c2_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-c4 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"bin_" -s 9 -c 3 -o gpurun_out/prof_bin_c2_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-c4 > /dev/null 2>&1
timeout 900 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_parity.py -q -x -k "boundary or empty or update or edge_sizes or unaligned or grow or closed_forms or long_row or hits or rwr or peer_exchange_single or understated or relabel_structure or partition or single_rank_acsr" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or bins_bitwise_rmat or long_row or window_rows or relabel_structure" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_racecheck_$TAG.txt
timeout 900 compute-sanitizer --tool synccheck python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or bins_bitwise_rmat or long_row or window_rows or update_insert or relabel_structure or hits_one" > gpurun_out/sanitizer_synccheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_synccheck_$TAG.txt
timeout 900 compute-sanitizer --tool initcheck python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes or bins_bitwise_rmat or spmv_float_rmat or update_insert or relabel_structure or pagerank_step_parity or single_rank_acsr" > gpurun_out/sanitizer_initcheck_$TAG.txt 2>&1; tail -n 3 gpurun_out/sanitizer_initcheck_$TAG.txt
ls gpurun_out | grep $TAG
