# session-2 A/B: shared-memory carveout shared by the binning and SpMV kernels (ACSR_CARVEOUT),
# and the L2-flush mode (write / write+read / none), graph-replayed steps (tools/graph_ab.py)
TAG=${1:-s2b}
mkdir -p gpurun_out
: > gpurun_out/carveout_ab_$TAG.jsonl
for rep in 1 2; do
for co in unset 28 100 0; do
  for wl in rmat10 rmat20 webgoogle; do
    if [ $co = unset ]; then timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/carveout_ab_$TAG.jsonl 2>>gpurun_out/carveout_ab_$TAG.err
    else ACSR_CARVEOUT=$co timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/carveout_ab_$TAG.jsonl 2>>gpurun_out/carveout_ab_$TAG.err; fi
  done
done
done
for fm in write+read none; do
  for wl in rmat10 rmat20 webgoogle; do
    GRAPH_AB_FLUSH=$fm timeout 300 python tools/graph_ab.py $wl 20 >> gpurun_out/carveout_ab_$TAG.jsonl 2>>gpurun_out/carveout_ab_$TAG.err
  done
done
cat gpurun_out/carveout_ab_$TAG.jsonl | cut -c1-250
