# round-2: CTA-batched unit claims + smaller units A/B; parity of the batched variant
TAG=${1:-r2o}
mkdir -p gpurun_out
ACSR_LIB_VARIANT=cb16w32 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "spmv or window or full_size or pagerank_step or bins" 2>&1 | tail -n 2
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" w32 cb16 cb16w32 cb32w32 cb16w32u1; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/ab_r2o.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append((r['t_bin_us'], r['t_spmv_us']))
for k,v in sorted(d.items()): print(k, v)
PY
