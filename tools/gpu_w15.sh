TAG=${1:-w15}
mkdir -p gpurun_out
for v in "" s1 x1 s1x1; do
  for wl in rmat20 livejournal; do COLPERM=1 ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1; done
done
cat gpurun_out/ab_$TAG.jsonl | cut -c1-200
timeout 600 ncu --section MemoryWorkloadAnalysis --section SpeedOfLight --clock-control none -k regex:spmv_kernel -s 4 -c 1 -o gpurun_out/prof_colperm_$TAG env COLPERM=1 python tools/spmv_ab.py rmat20 3 > /dev/null 2>&1
