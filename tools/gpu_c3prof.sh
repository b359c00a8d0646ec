# C3a/C3b SpMV profile + bench with NVML clocks
TAG=${1:-c3}
mkdir -p gpurun_out
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -1 gpurun_out/bench_$TAG.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['breakdown']['t_spmv_ms'], d['clocks'])"
for wl in webgoogle livejournal; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 3 -c 1 -o gpurun_out/prof_spmv_${wl}_$TAG python bench.py --workload $wl --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
done
ls gpurun_out | grep $TAG
