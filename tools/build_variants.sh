# Build compile-time A/B variants of libacsr.so (measurements only):
#   libacsr_<name>.so  with the -D flags listed below
set -e
cd "$(dirname "$0")/.."
L=paper_conf_sc_ashariseps14_b200/lib
NC=$(python -c "import __graft_entry__ as g; print(g.nccl_dirs()[0])")
NL=$(python -c "import __graft_entry__ as g; print(g.nccl_dirs()[1])")
F="-O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC -shared -cudart shared -I $NC"
build() { name=$1; shift; nvcc $F "$@" -o $L/libacsr_$name.so paper_conf_sc_ashariseps14_b200/csrc/*.cu -L $NL -l:libnccl.so.2 -Xlinker -rpath=$NL & }
for v in "$@"; do
  case $v in
    s1) build s1 -DACSR_STREAM_LD=1 ;;
    x1) build x1 -DACSR_X_LD=1 ;;
    s2) build s2 -DACSR_STREAM_LD=2 ;;
    x2) build x2 -DACSR_X_LD=2 ;;
    s2x2) build s2x2 -DACSR_STREAM_LD=2 -DACSR_X_LD=2 ;;
    st) build st -DACSR_SCHED_STATIC=1 ;;
    t256) build t256 -DACSR_SPMV_THREADS=256 ;;
    t512) build t512 -DACSR_SPMV_THREADS=512 ;;
    t256st) build t256st -DACSR_SPMV_THREADS=256 -DACSR_SCHED_STATIC=1 ;;
    nv) build nv -DACSR_NO_VEC=1 ;;
    br) build br -DACSR_BRANCHY_SUB=1 ;;
    nvbr) build nvbr -DACSR_NO_VEC=1 -DACSR_BRANCHY_SUB=1 ;;
    v256) build v256 -DACSR_VEC_MIN=256 ;;
    mb2) build mb2 -DACSR_MIN_BLOCKS=2 ;;
    u1) build u1 -DACSR_UNIT_SHIFT=1 ;;
    uw1) build uw1 -DACSR_UNIT_WARP_SHIFT=1 ;;
    pr) build pr -DACSR_PAIR_ROWS=1 ;;
    pruw1) build pruw1 -DACSR_PAIR_ROWS=1 -DACSR_UNIT_WARP_SHIFT=1 ;;
    uw2) build uw2 -DACSR_UNIT_WARP_SHIFT=2 ;;
    um1uw0) build um1uw0 -DACSR_UNIT_SHIFT=-1 ;;
    um1) build um1 -DACSR_UNIT_SHIFT=-1 ;;
    tile2k) build tile2k -DACSR_TILE_ROWS=2048 ;;
    tile512) build tile512 -DACSR_TILE_ROWS=512 ;;
    t512mb3) build t512mb3 -DACSR_SPMV_THREADS=512 -DACSR_MIN_BLOCKS=3 ;;
    t256mb6) build t256mb6 -DACSR_SPMV_THREADS=256 -DACSR_MIN_BLOCKS=6 ;;
    t256mb8) build t256mb8 -DACSR_SPMV_THREADS=256 -DACSR_MIN_BLOCKS=8 ;;
    v512) build v512 -DACSR_VEC_MIN=512 ;;
    v1024) build v1024 -DACSR_VEC_MIN=1024 ;;
    v512br) build v512br -DACSR_VEC_MIN=512 -DACSR_BRANCHY_SUB=1 ;;
    w0) build w0 -DACSR_WINDOW=0 ;;
    wu128) build wu128 -DACSR_WIN_UNIT_ROWS=128 ;;
    wu32) build wu32 -DACSR_WIN_UNIT_ROWS=32 ;;
    wu64) build wu64 -DACSR_WIN_UNIT_ROWS=64 ;;
    wg2) build wg2 -DACSR_WIN_G=2 ;;
    wg8) build wg8 -DACSR_WIN_G=8 ;;
    wb4) build wb4 -DACSR_WIN_MAX_BIN=4 ;;
    wb6) build wb6 -DACSR_WIN_MAX_BIN=6 ;;
    wb6u128) build wb6u128 -DACSR_WIN_MAX_BIN=6 -DACSR_WIN_UNIT_ROWS=128 ;;
    wb6u256) build wb6u256 -DACSR_WIN_MAX_BIN=6 -DACSR_WIN_UNIT_ROWS=256 ;;
    wu256) build wu256 -DACSR_WIN_UNIT_ROWS=256 ;;
    wp1) build wp1 -DACSR_WIN_PREFETCH=1 ;;
    l41) build l41 -DACSR_WIN_LDS4=1 ;;
    mw1) build mw1 -DACSR_MERGED_WARP_PATH=1 ;;
    td16) build td16 -DACSR_TAIL_DIV=16 ;;
    td0) build td0 -DACSR_TAIL_DIV=0 ;;
    uwr1) build uwr1 -DACSR_UPD_WARPREG=1 ;;
    us1) build us1 -DACSR_UPD_SUB=1 ;;
    sc256) build sc256 -DACSR_SCAN_THREADS=256 ;;
    td8) build td8 -DACSR_TAIL_DIV=8 ;;
    pf) build pf -DACSR_PF_UNIT=1 ;;
    ptp0) build ptp0 -DACSR_PEER_TILE_PUSH=0 ;;
    ws0) build ws0 -DACSR_WIN_SEGSCAN=0 ;;
    diag1) build diag1 -DACSR_DIAG=1 ;;
    sum1) build sum1 -DACSR_WIN_SUM4=0 ;;
    prof) build prof -DACSR_PROF=1 ;;
    tl) build tl -DACSR_TIMELINE=1 ;;
    s2wp) build s2wp -DACSR_WIN_PREFETCH=1 ;;
    s2lds4) build s2lds4 -DACSR_WIN_LDS4=1 ;;
    s2sum4) build s2sum4 -DACSR_WIN_SUM4=1 ;;
    s2pair) build s2pair -DACSR_PAIR_ROWS=1 ;;
    s2br) build s2br -DACSR_BRANCHY_SUB=1 ;;
    s2s1) build s2s1 -DACSR_STREAM_LD=1 ;;
    s2x1) build s2x1 -DACSR_X_LD=1 ;;
    s2mwp) build s2mwp -DACSR_MERGED_WARP_PATH=1 ;;
    d0off) build d0off -DACSR_DESC0=0 ;;
    d0pf) build d0pf -DACSR_DESC0=2 ;;
    s2td32) build s2td32 -DACSR_TAIL_DIV=32 ;;
    s2w64) build s2w64 -DACSR_WIN_UNIT_ROWS=64 ;;
    s2w256) build s2w256 -DACSR_WIN_UNIT_ROWS=256 ;;
    s2v512) build s2v512 -DACSR_VEC_MIN=512 ;;
    s2v2048) build s2v2048 -DACSR_VEC_MIN=2048 ;;
    s2um1) build s2um1 -DACSR_UNIT_SHIFT=-1 ;;
    s2u1) build s2u1 -DACSR_UNIT_SHIFT=1 ;;
    s2uw1) build s2uw1 -DACSR_UNIT_WARP_SHIFT=1 ;;
    s2wb4) build s2wb4 -DACSR_WIN_MAX_BIN=4 ;;
    s2cl2) build s2cl2 -DACSR_CLAIM_LATE=2 ;;
    s2g2) build s2g2 -DACSR_WIN_G=2 ;;
    s2bt128) build s2bt128 -DACSR_BIN_THREADS=128 ;;
    s2bt512) build s2bt512 -DACSR_BIN_THREADS=512 ;;
    s2t2k) build s2t2k -DACSR_TILE_ROWS=2048 ;;
    s2t512) build s2t512 -DACSR_TILE_ROWS=512 ;;
    l4) build l4 -DACSR_WIN_LANE4=1 ;;
    td2) build td2 -DACSR_TAIL_DIV=2 ;;
    td4x) build td4x -DACSR_TAIL_DIV=4 ;;
    l4s) build l4s -DACSR_WIN_LANE4=2 ;;
    tll4) build tll4 -DACSR_TIMELINE=1 -DACSR_WIN_LANE4=1 ;;
    g2) build g2 -DACSR_CLAIM_GUIDED=2 ;;
    g2w32) build g2w32 -DACSR_CLAIM_GUIDED=2 -DACSR_WIN_UNIT_ROWS=32 ;;
    g2w64) build g2w64 -DACSR_CLAIM_GUIDED=2 -DACSR_WIN_UNIT_ROWS=64 ;;
    g1w32) build g1w32 -DACSR_CLAIM_GUIDED=1 -DACSR_WIN_UNIT_ROWS=32 ;;
    g4w32) build g4w32 -DACSR_CLAIM_GUIDED=4 -DACSR_WIN_UNIT_ROWS=32 ;;
    g2w32na) build g2w32na -DACSR_CLAIM_GUIDED=2 -DACSR_WIN_UNIT_ROWS=32 -DACSR_GUIDED_AHEAD=0 ;;
    g2w32u) build g2w32u -DACSR_CLAIM_GUIDED=2 -DACSR_WIN_UNIT_ROWS=32 -DACSR_UNIT_SHIFT=-1 ;;
    tlg2w32) build tlg2w32 -DACSR_TIMELINE=1 -DACSR_CLAIM_GUIDED=2 -DACSR_WIN_UNIT_ROWS=32 ;;
    cb16) build cb16 -DACSR_CLAIM_BATCH=16 ;;
    cb16w32) build cb16w32 -DACSR_CLAIM_BATCH=16 -DACSR_WIN_UNIT_ROWS=32 ;;
    cb32w32) build cb32w32 -DACSR_CLAIM_BATCH=32 -DACSR_WIN_UNIT_ROWS=32 ;;
    cb16w32u1) build cb16w32u1 -DACSR_CLAIM_BATCH=16 -DACSR_WIN_UNIT_ROWS=32 -DACSR_UNIT_SHIFT=-1 ;;
    w32) build w32 -DACSR_WIN_UNIT_ROWS=32 ;;
    prs) build prs -DACSR_PR_STREAM_HINTS=1 ;;
    s1x1) build s1x1 -DACSR_STREAM_LD=1 -DACSR_X_LD=1 ;;
    pfs64) build pfs64 -DACSR_PF_START_TILES=64 ;;
    pfs256) build pfs256 -DACSR_PF_START_TILES=256 ;;
    rpl2) build rpl2 -DACSR_WIN_RPL=2 ;;
    rpl4) build rpl4 -DACSR_WIN_RPL=4 ;;
    rpl2g8) build rpl2g8 -DACSR_WIN_RPL=2 -DACSR_WIN_G=8 ;;
    rpl4g8) build rpl4g8 -DACSR_WIN_RPL=4 -DACSR_WIN_G=8 ;;
    da) build da -DACSR_DESC_AHEAD=1 ;;
    daw32) build daw32 -DACSR_DESC_AHEAD=1 -DACSR_WIN_UNIT_ROWS=32 ;;
    daw64) build daw64 -DACSR_DESC_AHEAD=1 -DACSR_WIN_UNIT_ROWS=64 ;;
    dawp) build dawp -DACSR_DESC_AHEAD=1 -DACSR_WIN_PREFETCH=1 ;;
    daw32wp) build daw32wp -DACSR_DESC_AHEAD=1 -DACSR_WIN_UNIT_ROWS=32 -DACSR_WIN_PREFETCH=1 ;;
    cl1) build cl1 -DACSR_CLAIM_LATE=1 ;;
    cl2) build cl2 -DACSR_CLAIM_LATE=2 ;;
    cl1w32) build cl1w32 -DACSR_CLAIM_LATE=1 -DACSR_WIN_UNIT_ROWS=32 ;;
    cl2w32) build cl2w32 -DACSR_CLAIM_LATE=2 -DACSR_WIN_UNIT_ROWS=32 ;;
    cl2w64) build cl2w64 -DACSR_CLAIM_LATE=2 -DACSR_WIN_UNIT_ROWS=64 ;;
    cl2um1) build cl2um1 -DACSR_CLAIM_LATE=2 -DACSR_UNIT_SHIFT=-1 ;;
    cl1um1) build cl1um1 -DACSR_CLAIM_LATE=1 -DACSR_UNIT_SHIFT=-1 ;;
    cl1w64) build cl1w64 -DACSR_CLAIM_LATE=1 -DACSR_WIN_UNIT_ROWS=64 ;;
    cl1u1) build cl1u1 -DACSR_CLAIM_LATE=1 -DACSR_UNIT_SHIFT=1 ;;
    cl1w256) build cl1w256 -DACSR_CLAIM_LATE=1 -DACSR_WIN_UNIT_ROWS=256 ;;
    t256mb4) build t256mb4 -DACSR_SPMV_THREADS=256 -DACSR_MIN_BLOCKS=4 ;;
    v768) build v768 -DACSR_VEC_MIN=768 ;;
    v2048) build v2048 -DACSR_VEC_MIN=2048 ;;
    cl0) build cl0 -DACSR_CLAIM_LATE=0 ;;
    cl0v512) build cl0v512 -DACSR_CLAIM_LATE=0 -DACSR_VEC_MIN=512 ;;
    cl2w256) build cl2w256 -DACSR_CLAIM_LATE=2 -DACSR_WIN_UNIT_ROWS=256 ;;
    noremote) build noremote -DACSR_DIAG=4 ;;
    noremote0) build noremote0 -DACSR_DIAG=4 -DACSR_PEER_TILE_PUSH=0 ;;
    pft32) build pft32 -DACSR_PF_TILES=32 ;;
    pft128) build pft128 -DACSR_PF_TILES=128 ;;
    pft320) build pft320 -DACSR_PF_TILES=320 ;;
    wg8d) build wg8d -DACSR_WIN_G=8 ;;
    wg6d) build wg6d -DACSR_WIN_G=6 ;;
    wg4d) build wg4d -DACSR_WIN_DYN_SMEM=1 ;;
    diag2) build diag2 -DACSR_DIAG=2 ;;
    diag12) build diag12 -DACSR_DIAG=3 ;;
    wu64s) build wu64s -DACSR_WIN_UNIT_ROWS=64 ;;
    wu32s) build wu32s -DACSR_WIN_UNIT_ROWS=32 ;;
    wb6s) build wb6s -DACSR_WIN_MAX_BIN=6 ;;
    t256mb5) build t256mb5 -DACSR_SPMV_THREADS=256 -DACSR_MIN_BLOCKS=5 ;;
    pft256mb5) build pft256mb5 -DACSR_PF_UNIT=1 -DACSR_SPMV_THREADS=256 -DACSR_MIN_BLOCKS=5 ;;
    pfwg8) build pfwg8 -DACSR_PF_UNIT=1 -DACSR_WIN_G=8 ;;
    td32) build td32 -DACSR_TAIL_DIV=32 ;;
    wu64) build wu64 -DACSR_WIN_UNIT_ROWS=64 ;;
    wu32) build wu32 -DACSR_WIN_UNIT_ROWS=32 ;;

    wg8) build wg8 -DACSR_WIN_G=8 ;;
    wb6) build wb6 -DACSR_WIN_MAX_BIN=6 ;;
  esac
done
wait
ls $L
