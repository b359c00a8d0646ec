# round-2: where the SpMV time goes -- diagnostic variants (no x gathers / no val loads / neither)
TAG=${1:-r2g}
mkdir -p gpurun_out
: > gpurun_out/diag_$TAG.jsonl
for rep in 1 2; do
for v in "" diag1 diag2 diag12; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/diag_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/diag_r2g.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
PY
for v in diag1; do
ACSR_LIB_VARIANT=$v timeout 600 ncu --set full --clock-control none -k regex:spmv_kernel -s 5 -c 1 -o gpurun_out/diag_${v}_c2_$TAG python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
done
ls gpurun_out | grep $TAG
