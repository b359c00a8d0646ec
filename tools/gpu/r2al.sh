# round-2: default bench line with graph-issued steps (+ the eager loop beside), C2 only
TAG=${1:-r2al}
mkdir -p gpurun_out
for fm in write write+read write write+read; do ACSR_BENCH_FLUSH=$fm timeout 900 python bench.py --no-c4 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo rc=$? $fm
tail -n 3 gpurun_out/bench_$TAG.err
python - gpurun_out/bench_$TAG.json <<'PY'
import json, sys
r = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
b = r["breakdown"]
print(r["value"], r["ms_per_step"], {k: b[k] for k in ("t_bin_ms", "t_spmv_ms", "t_step_eager_ms", "wall_s_eager_loop", "wall_s_timed_loop", "t_spmv_warm_back_to_back_ms")}, r["roofline"]["frac"], r["clocks"])
PY
done
