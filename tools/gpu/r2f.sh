# round-2: GPU suite on the segmented-scan windows; A/B segscan vs round-1 in-order window sums and window unit sizes; s26 relabel with sorted rows
TAG=${1:-r2f}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x -rf 2>&1 | tail -n 6 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" ws0 wu64s wu32s wb6s; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/ab_r2f.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
PY
timeout 900 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 --relabel --relabel-sort > gpurun_out/pr26_relabel_sort_$TAG.json 2>/dev/null; tail -c 900 gpurun_out/pr26_relabel_sort_$TAG.json
