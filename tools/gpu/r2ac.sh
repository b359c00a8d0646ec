TAG=${1:-r2ac}
mkdir -p gpurun_out
: > gpurun_out/step_ab_$TAG.jsonl
for rep in 1 2; do for v in "" pfs64 pfs256; do for wl in rmat20 webgoogle livejournal; do
  ACSR_LIB_VARIANT=$v timeout 300 python tools/step_ab.py $wl 2>/dev/null >> gpurun_out/step_ab_$TAG.jsonl
done; done; done
cat gpurun_out/step_ab_$TAG.jsonl
