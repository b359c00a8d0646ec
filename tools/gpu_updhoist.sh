TAG=${1:-updh}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -k "update or epoch or grow or capacity or graph or c_abi" 2>&1 | tail -n 2
timeout 600 python -m pytest tests/test_oracle_update.py -q 2>&1 | tail -n 1
for rep in 1 2; do for v in "" updold; do
ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload dynamic_mixed 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'n2_value_ms': l['value'], 't_update_ms': l['breakdown']['t_update_ms']}))" >> gpurun_out/ab_$TAG.jsonl
ACSR_LIB_VARIANT=$v timeout 900 python bench.py --workload dynamic 2>/dev/null | tail -n 1 | python -c "import sys,json; l=json.loads(sys.stdin.read()); print(json.dumps({'variant': '$v', 'c5_value_ms': l['value'], 't_update_ms': l['breakdown']['t_update_ms']}))" >> gpurun_out/ab_$TAG.jsonl
done; done
cat gpurun_out/ab_$TAG.jsonl
