TAG=${1:-w7}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -rf -x 2>&1 | tail -8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
for v in "ACSR_BIN_FUSED=1" "ACSR_BIN_FUSED=0"; do
  for wl in rmat20 livejournal; do env $v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1; done
done
cat gpurun_out/ab_$TAG.jsonl
ACSR_BIN_FUSED=1 timeout 900 python bench.py --workload pagerank --scale 26 --steps 3 --warmup 2 > gpurun_out/bench_pr26_$TAG.json 2>&1; tail -1 gpurun_out/bench_pr26_$TAG.json | cut -c1-700
timeout 300 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -x -k "edge_sizes" > gpurun_out/racecheck_$TAG.txt 2>&1; tail -3 gpurun_out/racecheck_$TAG.txt
