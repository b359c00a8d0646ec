# session-2: full GPU suite on the final code
TAG=${1:-s2y}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 4 > gpurun_out/pytest_gpu_$TAG.txt; cat gpurun_out/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
