TAG=${1:-td}
mkdir -p gpurun_out
ACSR_LIB_VARIANT=td16 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "not two_ranks and not peer and not row_split and not s26" 2>&1 | tail -n 2
for rep in 1 2; do
for v in "" td16 td8 td32; do
  for wl in webgoogle rmat20 livejournal rmat20_f32; do ACSR_LIB_VARIANT=$v timeout 120 python tools/spmv_ab.py $wl 40 >> gpurun_out/ab_$TAG.jsonl 2>/dev/null; done
done
done
python - $TAG <<'PY'
import json, sys
for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl"):
    if not l.startswith("{"): continue
    r=json.loads(l); print(r["env"].get("ACSR_LIB_VARIANT", "default"), r["wl"], r["t_bin_us"], r["t_spmv_us"], r["t_spmv_min_us"])
PY
