# ncu full captures of the SpMV launch, window build vs w0, three matrices
TAG=${1:-wp}
mkdir -p gpurun_out
for v in "" w0; do
for wl in rmat20 webgoogle livejournal; do
ACSR_LIB_VARIANT=$v timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 4 -c 1 -o gpurun_out/prof_${wl}_${v:-win}_$TAG python tools/spmv_ab.py $wl 2 > /dev/null 2>&1
done
done
ls gpurun_out | grep $TAG
