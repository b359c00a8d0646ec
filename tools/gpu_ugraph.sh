timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "graph or update or epoch or c_abi" 2>&1 | tail -n 3
timeout 900 python bench.py --workload dynamic 2>gpurun_out/ug.err | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(l['value'], json.dumps(l['breakdown']))"
tail -n 3 gpurun_out/ug.err
