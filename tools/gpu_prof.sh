# usage: bash tools/gpu_prof.sh <tag> [workload] [full]
TAG=${1:-r1}; WL=${2:-rmat20}; FULL=${3:-1}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf -x 2>&1 | tail -15 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python bench.py --steps 20 --warmup 5 --workload $WL > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
ACSR_XCACHE=1 timeout 300 python bench.py --steps 20 --warmup 5 --workload $WL --no-cpu-baseline > gpurun_out/bench_xc_$TAG.json 2>&1; cat gpurun_out/bench_xc_$TAG.json | cut -c1-600
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"spmv_kernel|bin_|xc_fill|update_|pagerank_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --workload $WL > /dev/null 2>&1
if [ "$FULL" = "1" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload $WL > gpurun_out/ncu_spmv_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"bin_" -s 3 -c 3 -o gpurun_out/prof_bin_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload $WL > gpurun_out/ncu_bin_$TAG.log 2>&1
fi
ls gpurun_out | grep $TAG
