TAG=${1:-w12}
mkdir -p gpurun_out
for rep in 1 2; do
for v in "" u1 um1 tile2k tile512; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
done
