# round-2: binning time vs matrix size (fixed cost vs per-row cost) for the launch paths
TAG=${1:-r2aj}
mkdir -p gpurun_out
: > gpurun_out/bin_curve_$TAG.jsonl
for envs in "X=0" "ACSR_PDL=0" "ACSR_BIN_SS=1" "ACSR_BIN_FUSED=1"; do
  for wl in rmat10 rmat14 rmat17 rmat20 rmat22; do
    env $envs timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"envs\": \"$envs\", /" >> gpurun_out/bin_curve_$TAG.jsonl
  done
done
TAG=$TAG python - <<'PY'
import json,os
for l in open('gpurun_out/bin_curve_%s.jsonl' % os.environ['TAG']):
    r=json.loads(l); print(r['envs'], r['wl'], r['n'], r['nnz'], r['t_bin_us'], r['t_spmv_us'])
PY
