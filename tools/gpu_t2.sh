timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "prefetch_views or unaligned" 2>&1 | tail -n 3
