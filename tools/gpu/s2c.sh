# session-2: per-unit timeline of the SpMV (ACSR_TIMELINE variant) on C2, C3a, C3b
TAG=${1:-s2c}
mkdir -p gpurun_out
: > gpurun_out/timeline_$TAG.jsonl
for wl in rmat20 webgoogle livejournal; do
  ACSR_LIB_VARIANT=tl timeout 300 python tools/spmv_timeline.py $wl >> gpurun_out/timeline_$TAG.jsonl 2>> gpurun_out/timeline_$TAG.err
done
tail -n 3 gpurun_out/timeline_$TAG.err
cut -c1-600 gpurun_out/timeline_$TAG.jsonl
