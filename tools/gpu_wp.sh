# A/B: window row-bound prefetch (default build) vs none (wp0), unit sizes
TAG=${1:-wp}
mkdir -p gpurun_out
for rep in 1 2; do
for v in "" wp0 wu256 wp0u256; do
  for wl in webgoogle rmat20 livejournal rmat20_f32; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
done
done
python - $TAG <<'PY'
import json, sys
rows=[json.loads(l) for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl") if l.startswith("{")]
for r in rows: print(r["env"].get("ACSR_LIB_VARIANT", "default"), r["wl"], r["t_bin_us"], r["t_spmv_us"], r["t_spmv_min_us"])
PY
