# session-2 final evidence: GPU suite, smoke, default bench (N=1, torchrun N=1, 2 ranks on one GPU), every
# bench line, ncu launch list + full captures (SpMV, binning), compute-sanitizer on the final code
TAG=${1:-s2z}
mkdir -p gpurun_out
bash tools/gpu/r2m.sh $TAG
bash tools/gpu/r2n.sh $TAG
