TAG=${1:-dyn}
mkdir -p gpurun_out
timeout 900 python bench.py --workload dynamic 2>gpurun_out/bench_dyn_$TAG.err | tail -1 > gpurun_out/bench_dyn_$TAG.jsonl
timeout 900 python bench.py --workload dynamic_mixed 2>>gpurun_out/bench_dyn_$TAG.err | tail -1 >> gpurun_out/bench_dyn_$TAG.jsonl
cut -c1-1500 gpurun_out/bench_dyn_$TAG.jsonl; tail -n 5 gpurun_out/bench_dyn_$TAG.err
