# session-2: default bench with the double-buffered resident-matrix e2e variant
TAG=${1:-s2v}
mkdir -p gpurun_out
timeout 600 python bench.py --no-c4 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 3 gpurun_out/bench_$TAG.err | cut -c1-300
python - <<PY
import json
d = json.loads(open("gpurun_out/bench_$TAG.json").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], json.dumps(d["e2e"]))
PY
