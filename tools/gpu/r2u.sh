TAG=${1:-r2u}
mkdir -p gpurun_out
timeout 1500 compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_parity.py -q -x -k "peer_exchange_two_ranks or peer_exchange_three or dist_pagerank_acsr_comm_two_ranks or c_abi or single_rank_acsr or exchange_layout or grow_layout" > gpurun_out/sanitizer_memcheck_multiproc_$TAG.txt 2>&1; tail -n 4 gpurun_out/sanitizer_memcheck_multiproc_$TAG.txt
timeout 1500 compute-sanitizer --tool racecheck --target-processes all python -m pytest tests/test_gpu_parity.py -q -x -k "peer_exchange_two_ranks and True" > gpurun_out/sanitizer_racecheck_peer_$TAG.txt 2>&1; tail -n 4 gpurun_out/sanitizer_racecheck_peer_$TAG.txt
