# PDL A/B (ACSR_PDL=0/1) on the bench step and the window variants; GPU tests first
TAG=${1:-pdl}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -rf 2>&1 | tail -5 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
for p in 1 0 1 0; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_PDL=$p timeout 300 python bench.py --workload $wl --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); b=d['breakdown']; print('pdl=$p', '$wl', d['ms_per_step'], b['t_bin_ms'], b['t_spmv_ms'], d['roofline']['frac'])"
  done
done
for v in w0 wu64; do
  for wl in rmat20 webgoogle livejournal; do
    ACSR_LIB_VARIANT=$v timeout 300 python bench.py --workload $wl --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); b=d['breakdown']; print('$v', '$wl', d['ms_per_step'], b['t_bin_ms'], b['t_spmv_ms'], d['roofline']['frac'])"
  done
done
for p in 1 0; do
ACSR_PDL=$p timeout 600 python bench.py --workload pagerank --scale 22 --steps 20 --warmup 3 2>/dev/null | tail -1 | cut -c1-300
done
