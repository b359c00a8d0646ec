timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "alternative_launch or global_search_path" 2>&1 | tail -n 3
