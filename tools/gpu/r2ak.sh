# round-2: graph-replayed timings (sub-tick resolution): late claims / vector threshold / binning re-checked
TAG=${1:-r2ak}
mkdir -p gpurun_out
: > gpurun_out/graph_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" cl0 cl0v512 v512 oldbin; do
  for wl in rmat10 rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 2>&1 | tail -n 1 >> gpurun_out/graph_ab_$TAG.jsonl
  done
done
done
TAG=$TAG python - <<'PY'
import json,os,collections
d=collections.defaultdict(list)
for l in open('gpurun_out/graph_ab_%s.jsonl' % os.environ['TAG']):
    try: r=json.loads(l)
    except Exception: print(l.strip()); continue
    d[(r['variant'] or 'base', r['wl'])].append((r['t_bin_us'], r['t_spmv_us'], r['t_step_us']))
for k,v in sorted(d.items()): print(k, v)
PY
