# A/B of SpMV variants; usage: bash tools/gpu_ab.sh <tag> [workloads...]
TAG=${1:-ab}; shift; WLS=${@:-rmat20}
mkdir -p gpurun_out
for wl in $WLS; do
  for v in "" "ACSR_SMEM_RESERVE=163840" "ACSR_SMEM_RESERVE=65536" "ACSR_XCACHE=1 ACSR_XC_BITS=14" "ACSR_XCACHE=1 ACSR_XC_BITS=13" "ACSR_XCACHE=1 ACSR_XC_BITS=12" "ACSR_XCACHE=1 ACSR_XC_BITS=11" "ACSR_XCACHE=1 ACSR_XC_BITS=12 ACSR_XC_MISS=1"; do
    env $v timeout 120 python tools/spmv_ab.py $wl >> gpurun_out/ab_$TAG.jsonl 2>&1
  done
done
cat gpurun_out/ab_$TAG.jsonl
