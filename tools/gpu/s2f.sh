# session-2 A/B: lane-4 window reduction (ACSR_WIN_LANE4) vs base, graph-replayed steps; parity of the variant
TAG=${1:-s2f}
mkdir -p gpurun_out
: > gpurun_out/lane4_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" l4; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/lane4_ab_$TAG.jsonl 2>>gpurun_out/lane4_ab_$TAG.err
  done
done
done
ACSR_LIB_VARIANT=l4 timeout 1200 python -m pytest tests -m gpu -q -k "not in_order_sums" 2>&1 | tail -n 4
ACSR_LIB_VARIANT=l4 timeout 300 python -m pytest tests -m gpu -q -k "in_order_sums" 2>&1 | tail -n 3
TAG=$TAG python - <<'PY'
import json, os
for l in open("gpurun_out/lane4_ab_%s.jsonl" % os.environ["TAG"]):
    d = json.loads(l)
    print(d["wl"].ljust(12), (d["variant"] or "base").ljust(6), d["t_bin_us"], d["t_spmv_us"], d["t_step_us"])
PY
