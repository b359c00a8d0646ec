TAG=${1:-ab3}
mkdir -p gpurun_out
for v in "" s1 x1 s1x1; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
cat gpurun_out/ab_$TAG.jsonl
timeout 300 python -m pytest tests/test_gpu_parity.py -q -k "dist or grow" 2>&1 | tail -3
