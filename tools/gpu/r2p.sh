TAG=${1:-r2p}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "hits or edge_cases or relabel_pagerank" 2>&1 | tail -n 2
for nc in 1048576 16777216; do timeout 300 ./tools/bin/stream_gather_bench $nc; done | tee gpurun_out/stream_gather_$TAG.jsonl
