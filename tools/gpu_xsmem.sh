TAG=${1:-xsmem}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "x_smem or pagerank or rwr or peer_exchange_single or c_abi" 2>&1 | tail -n 3
for rep in 1 2; do for xs in 0 8192 16384; do
timeout 600 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 --relabel --x-smem $xs 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'x_smem': $xs, 'wl': 's22_relabel', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 --relabel --x-smem $xs 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'x_smem': $xs, 'wl': 's26_relabel', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
done
timeout 600 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'x_smem': 0, 'wl': 's22_plain', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
done
cat gpurun_out/ab_$TAG.jsonl
