# round-2: with late claims as the default, re-check the geometry knobs (CTA size, tile, window max bin, merged warp path, vector threshold)
TAG=${1:-r2ag}
mkdir -p gpurun_out
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" t512 t256mb4 tile2k tile512 mw1 wb4 wb6 v256 v1024 wg2; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
TAG=$TAG python - <<'PY'
import json,collections,os
rows=[json.loads(l) for l in open('gpurun_out/ab_%s.jsonl' % os.environ['TAG']) if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append((r['t_bin_us'], r['t_spmv_us']))
for k,v in sorted(d.items()): print(k, v)
PY
