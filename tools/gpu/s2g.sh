# session-2 A/B: lane-4 window reduction with exact serial carries (ACSR_WIN_LANE4=2) vs base; full GPU suite on it; ncu of C3b
TAG=${1:-s2g}
mkdir -p gpurun_out
: > gpurun_out/lane4s_ab_$TAG.jsonl
for rep in 1 2; do
for v in "" l4s; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/lane4s_ab_$TAG.jsonl 2>>gpurun_out/lane4s_ab_$TAG.err
  done
done
done
TAG=$TAG python - <<'PY'
import json, os
for l in open("gpurun_out/lane4s_ab_%s.jsonl" % os.environ["TAG"]):
    d = json.loads(l)
    print(d["wl"].ljust(12), (d["variant"] or "base").ljust(6), d["t_bin_us"], d["t_spmv_us"], d["t_step_us"])
PY
ACSR_LIB_VARIANT=l4s timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -n 3
ACSR_LIB_VARIANT=l4s timeout 600 ncu --set full --clock-control none -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c3b_l4s_$TAG python tools/spmv_ab.py livejournal 3 > /dev/null 2>&1
ACSR_LIB_VARIANT=l4s timeout 600 ncu --set full --clock-control none -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c3a_l4s_$TAG python tools/spmv_ab.py webgoogle 3 > /dev/null 2>&1
ls gpurun_out | grep $TAG
