# session-2 A/B: capped tail division (at most 320 tail tiles) on the C4 PageRank step vs off
TAG=${1:-s2q}
mkdir -p gpurun_out
: > gpurun_out/c4_taildiv_cap_$TAG.jsonl
for rep in 1 2; do
for v in "" td0; do
  for rl in "" "--relabel"; do
    ACSR_LIB_VARIANT=$v timeout 600 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 $rl --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); d['variant']=sys.argv[1]; print(json.dumps(d))" "$v" >> gpurun_out/c4_taildiv_cap_$TAG.jsonl
  done
done
done
python - <<PY
import json
for l in open("gpurun_out/c4_taildiv_cap_$TAG.jsonl"):
    d = json.loads(l)
    print((d["variant"] or "base").ljust(8), d["config"]["workload"].ljust(45), d["ms_per_step"])
PY
