# A/B: L2 bulk prefetch of x at SpMV entry (default) vs off (ACSR_XPREFETCH=0)
TAG=${1:-xpf}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "rmat14 or boundary or unaligned or ragged or full_size_rmat20 or pagerank_step or empty" 2>&1 | tail -n 1
for rep in 1 2; do
for pf in 1 0; do
  for wl in rmat20 rmat20_f32 webgoogle livejournal; do ACSR_XPREFETCH=$pf timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
  ACSR_XPREFETCH=$pf timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'pf': '$pf', 'bench_value': l['value'], 't_bin': l['breakdown']['t_bin_ms'], 't_spmv': l['breakdown']['t_spmv_ms'], 'warm': l['breakdown']['t_spmv_warm_back_to_back_ms']}))" >> gpurun_out/ab_$TAG.jsonl
  ACSR_XPREFETCH=$pf timeout 300 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'pf': '$pf', 'pagerank_s22_ms': l['ms_per_step']}))" >> gpurun_out/ab_$TAG.jsonl
done
done
python - $TAG <<'PY'
import json, sys
for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl"):
    if not l.startswith("{"): continue
    r=json.loads(l)
    if "wl" in r: print("pf", r["env"].get("ACSR_XPREFETCH"), r["wl"], r["t_bin_us"], r["t_spmv_us"], r["t_spmv_min_us"])
    else: print(r)
PY
