TAG=${1:-r2z}
mkdir -p gpurun_out
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" s1 x1 s1x1; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/ab_r2z.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
PY
