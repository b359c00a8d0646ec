TAG=${1:-w5}
mkdir -p gpurun_out
timeout 900 python bench.py --workload dynamic_mixed > gpurun_out/bench_dynmix_$TAG.json 2>&1; tail -2 gpurun_out/bench_dynmix_$TAG.json
for v in "" nv br nvbr; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
cat gpurun_out/ab_$TAG.jsonl
