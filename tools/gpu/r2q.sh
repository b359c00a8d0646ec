TAG=${1:-r2q}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -rA -k "c5_full or edge_cases or hits or relabel_pagerank" --durations=6 2>&1 | tail -n 16
