TAG=${1:-r2v}
mkdir -p gpurun_out
: > gpurun_out/pr_ab_$TAG.jsonl
for rep in 1 2; do for v in "" prs; do
  for sc in 22 26; do
    ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload pagerank --scale $sc --steps 10 --warmup 3 2>/dev/null | tail -n 1 | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/pr_ab_$TAG.jsonl
    ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload pagerank --scale $sc --steps 10 --warmup 3 --relabel 2>/dev/null | tail -n 1 | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/pr_ab_$TAG.jsonl
  done
done; done
python - <<'PY'
import json
for l in open('gpurun_out/pr_ab_r2v.jsonl'):
    if not l.strip(): continue
    d=json.loads(l); print(d['variant'] or 'base', d['config']['workload'], d['ms_per_step'], d['breakdown'].get('cold_run_ms'))
PY
