# session-2 A/B: guided batch claims (ACSR_CLAIM_GUIDED) x window unit rows, graph-replayed steps,
# + timeline of the guided 32-row-window variant, + parity of the best candidates
TAG=${1:-s2d}
mkdir -p gpurun_out
: > gpurun_out/guided_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" g2 g2w32 g2w64 g1w32 g4w32 g2w32na g2w32u; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/guided_ab_$TAG.jsonl 2>>gpurun_out/guided_ab_$TAG.err
  done
done
done
: > gpurun_out/timeline_$TAG.jsonl
for wl in rmat20 webgoogle livejournal; do
  ACSR_LIB_VARIANT=tlg2w32 timeout 300 python tools/spmv_timeline.py $wl >> gpurun_out/timeline_$TAG.jsonl 2>> gpurun_out/timeline_$TAG.err
done
for v in g2w32 g2w64; do
  ACSR_LIB_VARIANT=$v timeout 900 python -m pytest tests -m gpu -q -x -k "full_size or property or window or plan or heavy" 2>&1 | tail -n 2
done
TAG=$TAG python - <<'PY'
import json
for l in open("gpurun_out/guided_ab_%s.jsonl" % __import__("os").environ.get("TAG","s2d")):
    d = json.loads(l)
    print(d["wl"].ljust(12), d["variant"].ljust(9), d["t_bin_us"], d["t_spmv_us"], d["t_step_us"])
PY
