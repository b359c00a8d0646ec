mkdir -p gpurun_out
timeout 300 ./tools/bin/gather_bench > gpurun_out/gather_bench.jsonl 2>&1; cat gpurun_out/gather_bench.jsonl
