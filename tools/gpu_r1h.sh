# session-3 verification of HEAD: gpu tests, smoke, default bench, launch list
TAG=${1:-r1h}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi_$TAG.txt
timeout 1500 python -m pytest tests -m gpu -q -rf 2>&1 | tail -8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -2
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -1 gpurun_out/bench_$TAG.json
for wl in rmat20_f32 webgoogle livejournal; do timeout 300 python bench.py --workload $wl --no-cpu-baseline 2>/dev/null | tail -1 >> gpurun_out/bench_lines_$TAG.jsonl; done
cut -c1-400 gpurun_out/bench_lines_$TAG.jsonl
