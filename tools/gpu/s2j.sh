# session-2 A/B: 4x smaller work units in the last 1/D tiles (ACSR_TAIL_DIV) under late claims, graph-replayed steps
TAG=${1:-s2j}
mkdir -p gpurun_out
: > gpurun_out/taildiv_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" td2 td4x td8 td16; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/taildiv_ab_$TAG.jsonl 2>>gpurun_out/taildiv_ab_$TAG.err
  done
done
done
python - <<PY
import json
for l in open("gpurun_out/taildiv_ab_$TAG.jsonl"):
    d = json.loads(l)
    print(d["wl"].ljust(12), (d["variant"] or "base").ljust(6), d["t_bin_us"], d["t_spmv_us"], d["t_step_us"])
PY
