TAG=${1:-peer3}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -x -k "peer or two_ranks or row_split" 2>&1 | tail -n 5
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
