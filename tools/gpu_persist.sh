# A/B: L2 persisting window over the hot prefix of x (ACSR_X_PERSIST_MB) on PageRank
TAG=${1:-persist}
mkdir -p gpurun_out
python -c "
import torch; p=torch.cuda.get_device_properties(0); print('L2', p.L2_cache_size, 'persist max', getattr(p,'persisting_l2_cache_max_size',None))"
for mb in 0 16 32 64; do
  ACSR_X_PERSIST_MB=$mb timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 --relabel 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'persist_mb': $mb, 'wl': 's26_relabel', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
  ACSR_X_PERSIST_MB=$mb timeout 900 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'persist_mb': $mb, 'wl': 's26', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
  ACSR_X_PERSIST_MB=$mb timeout 300 python bench.py --workload pagerank --scale 24 --steps 10 --warmup 3 --relabel 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'persist_mb': $mb, 'wl': 's24_relabel', 'ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
done
cat gpurun_out/ab_$TAG.jsonl
