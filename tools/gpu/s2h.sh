# session-2: does column hotness (hot L2 slices) cost gather rate?  + ncu slice balance of two cases
TAG=${1:-s2h}
mkdir -p gpurun_out
timeout 300 python tools/hot_slice_probe.py > gpurun_out/hot_slice_$TAG.json 2> gpurun_out/hot_slice_$TAG.err; cat gpurun_out/hot_slice_$TAG.json; tail -n 3 gpurun_out/hot_slice_$TAG.err
timeout 300 ncu --metrics lts__t_tag_requests.avg.pct_of_peak_sustained_elapsed,lts__t_tag_requests.max.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,gpu__time_duration.sum,l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:index --csv python tools/hot_slice_probe.py > gpurun_out/hot_slice_ncu_$TAG.csv 2>/dev/null
python - <<PY
import csv, collections
rows = [r for r in csv.reader(open("gpurun_out/hot_slice_ncu_$TAG.csv")) if len(r) > 10]
h = rows[0]
agg = collections.defaultdict(list)
for r in rows[1:]:
    agg[(r[h.index("ID")])].append((r[h.index("Metric Name")], r[h.index("Metric Value")]))
ids = sorted(agg, key=int)
# 25 launches per case, 8 cases: print the last launch of each case
for c in range(len(ids) // 25):
    print(c, dict(agg[ids[c * 25 + 24]]))
PY
