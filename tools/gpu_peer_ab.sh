# N1 peer step vs plain step at N=1: launch lists, bench lines, full ncu captures
TAG=${1:-peerab}
mkdir -p gpurun_out
for ex in nccl peer; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|peer_" --csv --log-file gpurun_out/launches_${ex}_$TAG.csv python bench.py --workload pagerank_dist --scale 22 --steps 8 --warmup 3 --exchange $ex > /dev/null 2>&1
timeout 600 python bench.py --workload pagerank_dist --scale 22 --steps 20 --warmup 3 --exchange $ex 2>/dev/null | tail -1 >> gpurun_out/bench_peer_$TAG.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_${ex}_step_$TAG python bench.py --workload pagerank_dist --scale 22 --steps 2 --warmup 3 --exchange $ex > /dev/null 2>&1
done
cut -c1-300 gpurun_out/bench_peer_$TAG.jsonl
ls gpurun_out | grep $TAG
