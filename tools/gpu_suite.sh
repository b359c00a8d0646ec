timeout 1800 python -m pytest tests/ -x -q -m gpu 2>&1 | tail -n 3 > gpurun_out/pytest_gpu_final.txt; cat gpurun_out/pytest_gpu_final.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
