# round-2: stream-ahead tile L2 prefetch A/B; peer remote-store counts (P = 2, 3); C5 SpMV traffic
TAG=${1:-r2l}
mkdir -p gpurun_out
: > gpurun_out/ab_$TAG.jsonl
for rep in 1 2; do
for v in "" pft32 pft128 pft320; do
  for wl in rmat20 webgoogle livejournal rmat20_f32; do
    ACSR_LIB_VARIANT=$v timeout 300 python tools/spmv_ab.py $wl 30 2>/dev/null | sed "s/^{/{\"variant\": \"$v\", /" >> gpurun_out/ab_$TAG.jsonl
  done
done
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/ab_r2l.jsonl') if l.strip()]
d=collections.defaultdict(list)
for r in rows: d[(r['variant'] or 'base', r['wl'])].append(r['t_spmv_us'])
for k,v in sorted(d.items()): print(k, v)
PY
for P in 2 3; do for v in "" ptp0 noremote noremote0; do
ACSR_PEER_TIMEOUT_MS=8000 ACSR_LIB_VARIANT=$v timeout 600 ncu --target-processes all --metrics l1tex__t_requests_pipe_lsu_mem_global_op_st.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum -k regex:spmv_kernel -c $((3*P)) --csv --log-file gpurun_out/ncu_peer_P${P}_${v:-tile}_$TAG.csv python tools/peer_steps.py $P 18 3 > /dev/null 2>&1
done; done
timeout 900 ncu --kernel-name-base mangled --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct -k regex:IdLb0ELb1ELb0ELb0ELb0E -s 6 -c 1 --csv --log-file gpurun_out/ncu_c5_$TAG.csv python bench.py --workload dynamic --steps 3 --warmup 3 --batches 6 > /dev/null 2>&1
grep -v "^==" gpurun_out/ncu_c5_$TAG.csv | cut -c 1-250
