# N1 peer-exchange path: GPU tests + single-rank bench lines (nccl vs peer exchange)
TAG=${1:-peer}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "peer or two_ranks or device_side" 2>&1 | tail -15 > gpurun_out/pytest_peer_$TAG.txt; cat gpurun_out/pytest_peer_$TAG.txt
for ex in nccl peer; do timeout 600 python bench.py --workload pagerank_dist --scale 22 --steps 20 --warmup 3 --exchange $ex 2>gpurun_out/bench_peer_$ex.err | tail -1 >> gpurun_out/bench_peer_$TAG.jsonl; done
cut -c1-600 gpurun_out/bench_peer_$TAG.jsonl
for f in gpurun_out/bench_peer_*.err; do tail -n 3 $f; done
