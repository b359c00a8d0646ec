TAG=${1:-upd}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"update_|bin_|relayout" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --workload dynamic_mixed > /dev/null 2>&1
python - <<'PY'
import csv
from collections import defaultdict
rows=[r for r in csv.reader(open("gpurun_out/launches_upd.csv")) if len(r)>10]
h=rows[0]; ki=h.index("Kernel Name"); vi=h.index("Metric Value")
d=defaultdict(list)
for r in rows[1:]: d[r[ki].split('(')[0][:50]].append(float(r[vi]))
for k,v in d.items(): print(k, len(v), "mean us", round(sum(v)/len(v)/1000,2), "max", round(max(v)/1000,2))
PY
