# round-2: new parity tests (full-size every row, s26 3 steps in full, HITS one step, overflow)
TAG=${1:-r2b}
mkdir -p gpurun_out
nproc > gpurun_out/nproc_$TAG.txt; free -g >> gpurun_out/nproc_$TAG.txt
timeout 2400 python -m pytest tests/test_gpu_parity.py -q -x -rA -k "every_row or hits_one_step or understated" --durations=10 2>&1 | tail -n 30 > gpurun_out/pytest_new_$TAG.txt; tail -n 15 gpurun_out/pytest_new_$TAG.txt
