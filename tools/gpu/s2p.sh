# session-2 A/B: first unit descriptor: loaded with the header (default build) vs off vs an L1 prefetch (ACSR_DESC0=2)
TAG=${1:-s2o}
mkdir -p gpurun_out
: > gpurun_out/desc0b_ab_$TAG.jsonl
for rep in 1 2 3; do
for v in "" d0off d0pf; do
  for wl in rmat20 webgoogle livejournal rmat20_f32 rmat14; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/desc0b_ab_$TAG.jsonl 2>>gpurun_out/desc0b_ab_$TAG.err
  done
done
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/desc0b_ab_$TAG.jsonl"):
    r = json.loads(l); d[(r["variant"] or "base", r["wl"])].append((r["t_bin_us"], r["t_spmv_us"], r["t_step_us"]))
for k in sorted(d): print(k[0].ljust(8), k[1].ljust(12), d[k])
PY
