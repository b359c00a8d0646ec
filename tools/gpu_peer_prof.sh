# sanitizer + ncu evidence for the N1 peer-exchange path
TAG=${1:-peerprof}
mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_parity.py -q -x -k "peer" > gpurun_out/sanitizer_memcheck_$TAG.txt 2>&1; tail -n 4 gpurun_out/sanitizer_memcheck_$TAG.txt
timeout 900 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -k "peer_exchange_single_rank" > gpurun_out/sanitizer_racecheck_$TAG.txt 2>&1; tail -n 4 gpurun_out/sanitizer_racecheck_$TAG.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|peer_" --csv --log-file gpurun_out/launches_peer_$TAG.csv python bench.py --workload pagerank_dist --scale 22 --steps 8 --warmup 3 --exchange peer > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel" --csv --log-file gpurun_out/launches_nccl_$TAG.csv python bench.py --workload pagerank_dist --scale 22 --steps 8 --warmup 3 --exchange nccl > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 6 -c 1 -o gpurun_out/prof_peer_step_$TAG python bench.py --workload pagerank_dist --scale 22 --steps 2 --warmup 3 --exchange peer > /dev/null 2>&1
ls -la gpurun_out | grep $TAG
