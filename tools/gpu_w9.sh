TAG=${1:-w9}
mkdir -p gpurun_out
for rep in 1 2; do
for v in "" mb2 t512mb3 t256mb6 t256mb8; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
done
cat gpurun_out/ab_$TAG.jsonl | cut -c1-200
