timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "three_ranks or peer_exchange_two" 2>&1 | tail -n 3
timeout 600 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 2>/dev/null | tail -n 1 | cut -c1-260
