# short-row window mapping: GPU parity + A/B against the per-bin Alg. 2 mapping
TAG=${1:-win}
mkdir -p gpurun_out
[ -n "$NOTEST" ] || timeout 1200 python -m pytest tests -m gpu -q -x -rf 2>&1 | tail -15 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
for v0 in ${VARIANTS:-base w0 wu128 wu32 wg2 wb4 wb6}; do
  v=$v0; [ "$v0" = base ] && v=""
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl ${REPS:-20} >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
TAG=$TAG python - <<'PY'
import json, os
TAG = os.environ['TAG']
for l in open("gpurun_out/ab_%s.jsonl" % TAG):
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d["wl"], d["env"], d["t_bin_us"], d["t_spmv_us"], d["t_spmv_min_us"], d.get("t_spmv_mean_us"), d["spmv_GBs"])
PY
