# refresh the round-1 ncu evidence for the current code: launch list of bench.py (C2),
# full captures of spmv_kernel (C2, C3a, C3b) and the three bin kernels (C2)
TAG=${1:-r1g}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv_kernel|bin_|update_|pagerank_|xc_|hits_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_c2_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"bin_" -s 9 -c 3 -o gpurun_out/prof_bin_c2_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
for wl in webgoogle livejournal rmat20_f32; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_${wl}_$TAG python bench.py --workload $wl --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_pr22_$TAG python bench.py --workload pagerank --scale 22 --steps 2 --warmup 3 > /dev/null 2>&1
ls -la gpurun_out | grep $TAG
