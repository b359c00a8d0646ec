# session-2 A/B: binning CTA size and tile rows (graph-replayed steps)
TAG=${1:-s2m}
mkdir -p gpurun_out
: > gpurun_out/bingeom_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" s2bt128 s2bt512 s2t2k s2t512; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/bingeom_ab_$TAG.jsonl 2>>gpurun_out/bingeom_ab_$TAG.err
  done
done
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/bingeom_ab_$TAG.jsonl"):
    r = json.loads(l); d[(r["variant"] or "base", r["wl"])].append((r["t_bin_us"], r["t_spmv_us"], r["t_step_us"]))
for k in sorted(d): print(k[0].ljust(8), k[1].ljust(12), d[k])
PY
