# session-2 env-knob re-check with the graph-replay timer: x L2 prefetch off, single cooperative binning launch, fused scan+scatter
TAG=${1:-s2n}
mkdir -p gpurun_out
: > gpurun_out/envknob_ab_$TAG.jsonl
for rep in 1 2; do
for e in "ACSR_NONE=1" "ACSR_XPREFETCH=0" "ACSR_BIN_FUSED=1" "ACSR_BIN_SS=1"; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    env $e timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/envknob_ab_$TAG.jsonl 2>>gpurun_out/envknob_ab_$TAG.err
  done
done
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/envknob_ab_$TAG.jsonl"):
    r = json.loads(l); d[(json.dumps(r["env"]), r["wl"])].append((r["t_bin_us"], r["t_spmv_us"], r["t_step_us"]))
for k in sorted(d): print(k[0].ljust(28), k[1].ljust(12), d[k])
PY
