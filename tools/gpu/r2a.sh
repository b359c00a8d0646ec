# round-2 baseline: GPU suite, default bench line, gather microbenchmark + ncu of it
TAG=${1:-r2a}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi_$TAG.txt
timeout 300 ./tools/bin/gather_bench > gpurun_out/gather_bench_$TAG.jsonl 2> gpurun_out/gather_bench_$TAG.err; tail -n 3 gpurun_out/gather_bench_$TAG.err
timeout 600 ncu --set full --clock-control none -k regex:gather -o gpurun_out/gather_$TAG ./tools/bin/gather_bench ncu > gpurun_out/gather_ncu_$TAG.log 2>&1; tail -n 2 gpurun_out/gather_ncu_$TAG.log
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-400
timeout 1800 python -m pytest tests -m gpu -q -x 2>&1 | tail -n 4 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
