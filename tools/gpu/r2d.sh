# round-2: SpMV A/B (L2 prefetch of unit runs, 40 warps/SM), relabel test + s26 relabel bench, 2-rank torchrun debug
TAG=${1:-r2d}
mkdir -p gpurun_out
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" pf t256mb5 pft256mb5; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json
rows=[json.loads(l) for l in open('gpurun_out/ab_r2d.jsonl') if l.strip()]
for r in rows: print(r['variant'] or 'base', r['wl'], r['t_bin_us'], r['t_spmv_us'], r['t_spmv_min_us'])
PY
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "relabel" 2>&1 | tail -n 3
timeout 900 python bench.py --workload pagerank --scale 26 --steps 10 --warmup 3 --relabel > gpurun_out/pr26_relabel_$TAG.json 2>gpurun_out/pr26_relabel_$TAG.err; tail -c 1500 gpurun_out/pr26_relabel_$TAG.json; tail -n 3 gpurun_out/pr26_relabel_$TAG.err
PYTHONUNBUFFERED=1 ACSR_BENCH_WATCHDOG=500 NCCL_DEBUG=WARN ACSR_SHARED_GPU_TEST=1 ACSR_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --no-cpu-baseline --steps 10 --c4-scale 22 > gpurun_out/bench_tr2_$TAG.json 2> gpurun_out/bench_tr2_$TAG.err; tail -c 2000 gpurun_out/bench_tr2_$TAG.json; grep -v "UserWarning\|sparse_csr_tensor" gpurun_out/bench_tr2_$TAG.err | tail -n 40
