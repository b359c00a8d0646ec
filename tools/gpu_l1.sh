TAG=${1:-l1}
for rep in 1 2; do for rs in 0 24576 60000; do
for wl in rmat20 webgoogle livejournal; do ACSR_SMEM_RESERVE=$rs timeout 120 python tools/spmv_ab.py $wl 40 2>/dev/null | python -c "import sys,json; r=json.loads(sys.stdin.read()); print(json.dumps({'reserve': $rs, 'wl': r['wl'], 't_spmv_us': r['t_spmv_us']}))" >> gpurun_out/ab_$TAG.jsonl; done
done; done
cat gpurun_out/ab_$TAG.jsonl
