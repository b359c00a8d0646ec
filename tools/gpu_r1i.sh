# full GPU suite + headline bench lines (session 3)
TAG=${1:-r1i}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 8 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -n 2
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -n 1 gpurun_out/bench_$TAG.json | cut -c1-400
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 2>/dev/null | tail -n 1 | cut -c1-300
