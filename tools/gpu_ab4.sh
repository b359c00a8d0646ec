TAG=${1:-ab4}
mkdir -p gpurun_out
for v in "" st t256 t512 t256st s2 x2 s2x2; do
  for wl in rmat20 livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
cat gpurun_out/ab_$TAG.jsonl
for v in "" x2 s2x2; do
  ACSR_LIB_VARIANT=$v timeout 600 python bench.py --workload pagerank --scale 26 --steps 5 --warmup 2 > gpurun_out/pr26_${v}_$TAG.json 2>&1; tail -1 gpurun_out/pr26_${v}_$TAG.json | cut -c1-420
done
