TAG=${1:-w13}
mkdir -p gpurun_out
for rep in 1 2; do
for v in "" uw1 uw2 um1 pr pruw1; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
done
