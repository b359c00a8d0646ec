# session-2 final-code ncu DRAM traffic of the C4 step (plain, relabelled) and the C5 SpMV
TAG=${1:-s2s}
mkdir -p gpurun_out
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_requests_srcunit_tex_op_read.sum,l1tex__t_sector_hit_rate.pct,l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 900 ncu --metrics $M --clock-control none -k regex:spmv_kernel -s 4 -c 1 --csv --log-file gpurun_out/ncu_c4_plain_$TAG.csv python bench.py --workload pagerank --scale 26 --steps 2 --warmup 3 > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:spmv_kernel -s 4 -c 1 --csv --log-file gpurun_out/ncu_c4_relabel_$TAG.csv python bench.py --workload pagerank --scale 26 --steps 2 --warmup 3 --relabel > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:spmv_kernel -s 40 -c 1 --csv --log-file gpurun_out/ncu_c5_$TAG.csv python bench.py --workload dynamic --steps 3 --warmup 3 --batches 6 > /dev/null 2>&1
for f in gpurun_out/ncu_c*_$TAG.csv; do echo "== $f"; grep -v "^==PROF==" $f | cut -c1-300 | tail -n 9; done
