TAG=${1:-r2i}
mkdir -p gpurun_out
: > gpurun_out/prof_$TAG.jsonl
for wl in rmat20 webgoogle livejournal; do ACSR_LIB_VARIANT=prof timeout 300 python tools/spmv_prof.py $wl 10 >> gpurun_out/prof_$TAG.jsonl 2>gpurun_out/prof_$TAG.err; done
cat gpurun_out/prof_$TAG.jsonl; tail -3 gpurun_out/prof_$TAG.err
