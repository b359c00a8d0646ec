# session-2: property tests (single-tile and multi-tile) on the final code
TAG=${1:-s2x}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -k "property" 2>&1 | tail -n 5
