# fused scan+scatter (default) vs separate scan kernel (ACSR_BIN_SS=0)
TAG=${1:-ss}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -n 2
ACSR_BIN_SS=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "bins or rmat14 or boundary" 2>&1 | tail -n 1
for rep in 1 2; do
for ss in 1 0; do
  for wl in rmat20 webgoogle livejournal; do ACSR_BIN_SS=$ss timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
  ACSR_BIN_SS=$ss timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'ss': '$ss', 'bench_value': l['value'], 't_bin': l['breakdown']['t_bin_ms'], 't_spmv': l['breakdown']['t_spmv_ms']}))" >> gpurun_out/ab_$TAG.jsonl
  ACSR_BIN_SS=$ss timeout 600 python bench.py --workload pagerank --scale 26 --steps 3 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'ss': '$ss', 's26_t_bin_ms': l['breakdown']['t_bin_ms']}))" >> gpurun_out/ab_$TAG.jsonl
done
done
python - $TAG <<'PY'
import json, sys
for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl"):
    if not l.startswith("{"): continue
    r=json.loads(l)
    if "wl" in r: print("ss", r["env"].get("ACSR_BIN_SS"), r["wl"], r["t_bin_us"], r["t_spmv_us"])
    else: print(r)
PY
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
