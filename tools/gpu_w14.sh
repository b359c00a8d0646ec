TAG=${1:-w14}
mkdir -p gpurun_out
for v in "COLPERM=0" "COLPERM=1"; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do env $v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1; done
done
cat gpurun_out/ab_$TAG.jsonl
