timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "hits" 2>&1 | tail -n 1
timeout 300 python bench.py --workload hits 2>/dev/null | tail -n 1 > gpurun_out/bench_hits2.jsonl; cut -c1-400 gpurun_out/bench_hits2.jsonl
