TAG=${1:-usub}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "update or epoch or grow or capacity or dynamic or c_abi" 2>&1 | tail -n 3
ACSR_LIB_VARIANT=us0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "update or epoch" 2>&1 | tail -n 1
for rep in 1 2; do for v in "" us0; do
ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload dynamic_mixed 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'n2_value_ms': l['value'], 't_update_ms': l['breakdown']['t_update_ms']}))" >> gpurun_out/ab_$TAG.jsonl
ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload dynamic 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'c5_value_ms': l['value'], 't_update_ms': l['breakdown']['t_update_ms']}))" >> gpurun_out/ab_$TAG.jsonl
done; done
cat gpurun_out/ab_$TAG.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"update_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --workload dynamic_mixed > /dev/null 2>&1
python - <<'PY'
import csv
from collections import defaultdict
rows=[r for r in csv.reader(open("gpurun_out/launches_usub.csv")) if len(r)>10]
h=rows[0]; ki=h.index("Kernel Name"); vi=h.index("Metric Value")
d=defaultdict(list)
for r in rows[1:]: d[r[ki].split('(')[0][:50]].append(float(r[vi]))
for k,v in d.items(): print(k, len(v), "mean us", round(sum(v)/len(v)/1000,2), "max", round(max(v)/1000,2))
PY
