# session-2 geometry re-check with the precise graph-replay timer (tail division on by default)
TAG=${1:-s2l}
mkdir -p gpurun_out
: > gpurun_out/geom_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" s2td32 s2w64 s2w256 s2v512 s2v2048 s2um1 s2u1 s2uw1 s2wb4 s2cl2 s2g2; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/geom_ab_$TAG.jsonl 2>>gpurun_out/geom_ab_$TAG.err
  done
done
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/geom_ab_$TAG.jsonl"):
    r = json.loads(l); d[(r["variant"] or "base", r["wl"])].append(r["t_step_us"])
for k in sorted(d): print(k[0].ljust(8), k[1].ljust(12), d[k])
PY
