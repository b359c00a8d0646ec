TAG=${1:-w6}
mkdir -p gpurun_out
for rep in 1 2; do
for v in "" nv v256 v512 v1024 v512br; do
  for wl in rmat20 livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
done
cat gpurun_out/ab_$TAG.jsonl
