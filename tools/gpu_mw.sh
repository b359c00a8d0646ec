# A/B: merged heavy/warp-per-row path (default) vs separate paths (mw0)
TAG=${1:-mw}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -n 2
for rep in 1 2; do
for v in "" mw0; do
  for wl in rmat20 livejournal webgoogle; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
  ACSR_LIB_VARIANT=$v timeout 300 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'pagerank_s22_ms_per_iter': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
  ACSR_LIB_VARIANT=$v timeout 600 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'pagerank_s26_ms_per_iter': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
done
done
python - $TAG <<'PY'
import json, sys
for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl"):
    if not l.startswith("{"): continue
    r=json.loads(l)
    if "wl" in r: print(r["env"].get("ACSR_LIB_VARIANT", "default"), r["wl"], r["t_bin_us"], r["t_spmv_us"], r["t_spmv_min_us"])
    else: print(r)
PY
