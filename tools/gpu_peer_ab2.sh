TAG=${1:-peerab2}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "peer or two_ranks" 2>&1 | tail -n 3
for ex in nccl peer; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|peer_" --csv --log-file gpurun_out/launches_${ex}_$TAG.csv python bench.py --workload pagerank_dist --scale 22 --steps 8 --warmup 3 --exchange $ex > /dev/null 2>&1
timeout 600 python bench.py --workload pagerank_dist --scale 22 --steps 20 --warmup 3 --exchange $ex 2>/dev/null | tail -1 >> gpurun_out/bench_peer_$TAG.jsonl
done
timeout 600 python bench.py --workload pagerank --scale 22 --steps 10 --warmup 3 2>/dev/null | tail -1 >> gpurun_out/bench_peer_$TAG.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_peer_step_$TAG python bench.py --workload pagerank_dist --scale 22 --steps 2 --warmup 3 --exchange peer > /dev/null 2>&1
cut -c1-300 gpurun_out/bench_peer_$TAG.jsonl
