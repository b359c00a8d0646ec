# session-2: default bench with the double-buffered e2e loop (+ the from-host tests)
TAG=${1:-s2u}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -k "host or capi or smoke" 2>&1 | tail -n 2
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 3 gpurun_out/bench_$TAG.err
python - <<PY
import json
d = json.loads(open("gpurun_out/bench_$TAG.json").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], json.dumps(d["e2e"]))
PY
