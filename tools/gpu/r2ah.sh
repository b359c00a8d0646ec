# round-2: vectorised-row threshold (ACSR_VEC_MIN) under late claims; PageRank s26 for the candidate
TAG=${1:-r2ah}
mkdir -p gpurun_out
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2 3; do
for v in "" v768 v1024 v2048; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
: > gpurun_out/pr_$TAG.jsonl
for v in "" v1024 v2048; do
  for rl in "" "--relabel"; do
    ACSR_LIB_VARIANT=$v timeout 600 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 --no-cpu-baseline $rl 2>/dev/null | tail -n 1 | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/pr_$TAG.jsonl
  done
done
TAG=$TAG python - <<'PY'
import json,collections,os
rows=[json.loads(l) for l in open('gpurun_out/ab_%s.jsonl' % os.environ['TAG']) if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
for l in open('gpurun_out/pr_%s.jsonl' % os.environ['TAG']):
    r=json.loads(l); print(r.get('variant'), r['config'].get('relabel'), r['value'], r['unit'], r.get('ms_per_step'))
PY
