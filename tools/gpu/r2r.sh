# round-2: wide short-row windows (rows per lane 2/4, groups 4/8): parity + A/B
TAG=${1:-r2r}
mkdir -p gpurun_out
for v in rpl2 rpl4g8; do ACSR_LIB_VARIANT=$v timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "window or spmv_float or integer_bitwise or full_size or pagerank_step or boundary or ragged" 2>&1 | tail -n 1; done
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" rpl2 rpl4 rpl2g8 rpl4g8; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/ab_r2r.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
PY
