# Build compile-time A/B variants of libacsr.so (measurements only):
#   libacsr_<name>.so  with the -D flags listed below
set -e
cd "$(dirname "$0")/.."
L=paper_conf_sc_ashariseps14_b200/lib
F="-O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC -shared -cudart shared"
build() { name=$1; shift; nvcc $F "$@" -o $L/libacsr_$name.so paper_conf_sc_ashariseps14_b200/csrc/*.cu; }
build s1 -DACSR_STREAM_LD=1
build x1 -DACSR_X_LD=1
build s1x1 -DACSR_STREAM_LD=1 -DACSR_X_LD=1
ls $L
