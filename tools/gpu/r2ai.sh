# round-2: binning with segment-parallel scans (2 barriers per tile instead of 8, no serial per-bin loops) vs the previous binning
TAG=${1:-r2ai}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "bin or full_size or c5 or edge or relabel or grow or update" 2>&1 | tail -n 2
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2 3; do
for v in "" oldbin; do
  for wl in rmat20 webgoogle livejournal; do
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
for v in "" oldbin; do
ACSR_LIB_VARIANT=$v ncu --metrics gpu__time_duration.sum --clock-control none -k regex:bin_ -c 12 --csv python tools/spmv_ab.py rmat20 3 2>/dev/null > gpurun_out/bin_launches_${TAG}_$v.csv
python - gpurun_out/bin_launches_${TAG}_$v.csv <<'PY'
import csv, sys, collections
d = collections.defaultdict(list)
for r in csv.reader(open(sys.argv[1])):
    if len(r) > 14 and r[12] == 'gpu__time_duration.sum': d[r[4].split('(')[0]].append(float(r[14]))
print(sys.argv[1], {k: round(sum(v) / len(v)) for k, v in d.items()})
PY
done
