TAG=${1:-f32}
for sr in window alg2 window alg2; do
  for wl in rmat20 rmat20_f32 webgoogle livejournal; do
    SHORT_ROWS=$sr timeout 120 python tools/spmv_ab.py $wl 60 >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
python - <<PY
import json
for l in open("gpurun_out/ab_$TAG.jsonl"):
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d["wl"], d["env"], d["t_bin_us"], d["t_spmv_us"], d["t_spmv_min_us"], d.get("t_spmv_mean_us"), d["spmv_GBs"])
PY
