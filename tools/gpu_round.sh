set -x
mkdir -p gpurun_out
nvidia-smi -L; nproc; lscpu | grep "Model name"
timeout 900 python -m pytest tests -m gpu -q -rf 2>&1 | tail -40 > gpurun_out/pytest_gpu.txt; cat gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -5
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err; cat gpurun_out/bench1.json; tail -5 gpurun_out/bench1.err
