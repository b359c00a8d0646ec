TAG=${1:-binfin}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -n 2
ACSR_BIN_SS=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "bins or rmat14 or boundary" 2>&1 | tail -n 1
ACSR_BIN_FUSED=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "bins or rmat14 or boundary" 2>&1 | tail -n 1
for rep in 1 2 3; do for v in "" binprev; do
  for wl in rmat20 webgoogle livejournal; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 2>/dev/null | python -c "import sys,json; r=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'wl': r['wl'], 't_bin_us': r['t_bin_us'], 't_spmv_us': r['t_spmv_us']}))" >> gpurun_out/ab_$TAG.jsonl; done
  ACSR_LIB_VARIANT=$v timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'bench_value': l['value'], 't_bin': l['breakdown']['t_bin_ms'], 't_spmv': l['breakdown']['t_spmv_ms']}))" >> gpurun_out/ab_$TAG.jsonl
done; done
cat gpurun_out/ab_$TAG.jsonl
