TAG=${1:-bins}
mkdir -p gpurun_out
timeout 300 python tools/spmv_bins.py > gpurun_out/bins_$TAG.jsonl 2>&1
cat gpurun_out/bins_$TAG.jsonl
for v in "" "ACSR_XCACHE=1"; do env $v timeout 120 python tools/spmv_ab.py rmat20 >> gpurun_out/ab_$TAG.jsonl 2>&1; done
cat gpurun_out/ab_$TAG.jsonl
timeout 300 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"spmv_kernel|bin_|xc_" --csv --log-file gpurun_out/launches_nc_$TAG.csv python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
