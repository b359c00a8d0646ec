timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "plain_c or e2e" 2>&1 | tail -n 3
timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | tail -n 1 > gpurun_out/bench_capi.json; python -c "
import json; l=json.loads(open('gpurun_out/bench_capi.json').read()); print(l['value'], json.dumps(l['e2e']))"
