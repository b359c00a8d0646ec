# session-2: ncu --set full of the web-Google-like (C3a) and LiveJournal-like (C3b) SpMV on the current code
TAG=${1:-s2e}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c3a_$TAG python tools/spmv_ab.py webgoogle 3 > gpurun_out/ncu_c3a_$TAG.log 2>&1; tail -n 2 gpurun_out/ncu_c3a_$TAG.log
timeout 600 ncu --set full --clock-control none -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c3b_$TAG python tools/spmv_ab.py livejournal 3 > gpurun_out/ncu_c3b_$TAG.log 2>&1; tail -n 2 gpurun_out/ncu_c3b_$TAG.log
ls -la gpurun_out | grep $TAG
