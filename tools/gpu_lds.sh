TAG=${1:-lds}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "window or powerlaw or boundary or rmat14 or ragged" 2>&1 | tail -n 2
for rep in 1 2; do
for v in "" l40 wu64 wu32; do
  for wl in webgoogle rmat20 livejournal rmat20_f32; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
done
done
python - $TAG <<'PY'
import json, sys
rows=[json.loads(l) for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl") if l.startswith("{")]
for r in rows: print(r["env"].get("ACSR_LIB_VARIANT", "default"), r["wl"], r["t_bin_us"], r["t_spmv_us"], r["t_spmv_min_us"])
PY
