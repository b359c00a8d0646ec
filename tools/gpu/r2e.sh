# round-2: peer tile push (tests + A/B vs per-row pushes, P = 2, 3 on one GPU), source-level ncu of C2 / C3a SpMV
TAG=${1:-r2e}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "peer or dist or update_graph" 2>&1 | tail -n 3
: > gpurun_out/peer_ab_$TAG.jsonl
for rep in 1 2; do for P in 2 3; do for v in "" ptp0; do
  ACSR_LIB_VARIANT=$v timeout 300 python tools/peer_steps.py $P 22 20 2>/dev/null | tail -n 1 >> gpurun_out/peer_ab_$TAG.jsonl
done; done; done
cat gpurun_out/peer_ab_$TAG.jsonl
for wl in rmat20 webgoogle; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:spmv_kernel -s 5 -c 1 -o gpurun_out/src_${wl}_$TAG python tools/spmv_ab.py $wl 3 > /dev/null 2>&1; ls -la gpurun_out/src_${wl}_$TAG.ncu-rep
done
