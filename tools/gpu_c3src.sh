TAG=${1:-c3src}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 4 -c 1 -o gpurun_out/prof_webgoogle_$TAG python tools/spmv_ab.py webgoogle 2 > /dev/null 2>&1
ls gpurun_out | grep $TAG
