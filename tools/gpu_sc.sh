TAG=${1:-sc}
mkdir -p gpurun_out
ACSR_LIB_VARIANT=sc256 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "bins or rmat14 or boundary or edge_sizes" 2>&1 | tail -n 1
for rep in 1 2 3; do for v in "" sc256; do
  for wl in rmat20 livejournal; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 2>/dev/null | python -c "import sys,json; r=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'wl': r['wl'], 't_bin_us': r['t_bin_us']}))" >> gpurun_out/ab_$TAG.jsonl; done
  ACSR_LIB_VARIANT=$v timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'bench_value': l['value'], 't_bin': l['breakdown']['t_bin_ms']}))" >> gpurun_out/ab_$TAG.jsonl
done; done
cat gpurun_out/ab_$TAG.jsonl
