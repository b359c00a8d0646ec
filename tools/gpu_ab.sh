# A/B of SpMV variants; usage: bash tools/gpu_ab.sh <tag> [workloads...]
TAG=${1:-ab}; shift; WLS=${@:-rmat20}
mkdir -p gpurun_out
for wl in $WLS; do
  timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  ACSR_NO_XCACHE=1 timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  ACSR_XC_MISS=1 timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
done
cat gpurun_out/ab_$TAG.jsonl
timeout 300 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"spmv_kernel|bin_|xc_" --csv --log-file gpurun_out/launches_nc_$TAG.csv python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
