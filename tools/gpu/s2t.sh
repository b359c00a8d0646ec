# session-2 re-check of round-1/2 compile knobs with the graph-replay timer (final code, tail division on)
TAG=${1:-s2t}
mkdir -p gpurun_out
: > gpurun_out/knobs_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" s2wp s2lds4 s2sum4 s2pair s2br s2s1 s2x1 s2mwp; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/knobs_ab_$TAG.jsonl 2>>gpurun_out/knobs_ab_$TAG.err
  done
done
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/knobs_ab_$TAG.jsonl"):
    r = json.loads(l); d[(r["variant"] or "base", r["wl"])].append(r["t_step_us"])
for k in sorted(d): print(k[0].ljust(8), k[1].ljust(12), d[k])
PY
