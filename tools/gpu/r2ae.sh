# round-2: late unit claims (balance at 1-2 units per warp) x unit size A/B
TAG=${1:-r2ae}
mkdir -p gpurun_out
for v in cl2 cl2w32; do
ACSR_LIB_VARIANT=$v timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "spmv or window or full_size or pagerank_step or bins" 2>&1 | tail -n 1
done
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" cl1 cl2 cl1w32 cl2w32 cl2w64 cl2um1; do
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
