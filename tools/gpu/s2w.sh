# session-2 A/B: largest x bulk-prefetched into L2 at kernel entry (ACSR_XPREFETCH_MAX_MB 32 default / 48 / 96)
TAG=${1:-s2w}
mkdir -p gpurun_out
: > gpurun_out/xpf_ab_$TAG.jsonl
for rep in 1 2; do
for mb in 32 48 96; do
  for wl in livejournal rmat20 webgoogle; do
    ACSR_XPREFETCH_MAX_MB=$mb timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/xpf_ab_$TAG.jsonl 2>>gpurun_out/xpf_ab_$TAG.err
  done
done
done
for mb in 32 96; do
  ACSR_XPREFETCH_MAX_MB=$mb timeout 600 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -n 1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('pagerank s22', sys.argv[1], d['ms_per_step'])" $mb
done
python - <<PY
import json, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/xpf_ab_$TAG.jsonl"):
    r = json.loads(l); d[(r["env"].get("ACSR_XPREFETCH_MAX_MB"), r["wl"])].append((r["t_spmv_us"], r["t_step_us"]))
for k in sorted(d): print(k[0], k[1].ljust(12), d[k])
PY
