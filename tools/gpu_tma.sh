mkdir -p gpurun_out
timeout 60 ./tools/bin/tma_gather_bench > gpurun_out/tma_gather.jsonl 2>&1; echo rc=$?; cat gpurun_out/tma_gather.jsonl
