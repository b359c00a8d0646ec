// acsr_internal.cuh -- constants, plan-workspace layout and small device helpers
// shared by the libacsr.so translation units.  sm_100a only.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/acsr.h"

namespace acsr {

// ---------------------------------------------------------------- binning tiles
// acsr_bin processes the rows in tiles of TILE_ROWS rows (one CTA per tile, rounds
// of 256 rows in row order).  The per-(bin, tile) counts double as the row-space
// locality unit of the SpMV work map.
#ifndef ACSR_BIN_THREADS
#define ACSR_BIN_THREADS 256  // threads per binning CTA (A/B knob)
#endif
constexpr int BIN_THREADS = ACSR_BIN_THREADS;
#ifndef ACSR_TILE_ROWS
#define ACSR_TILE_ROWS 1024
#endif
constexpr int TILE_ROWS = ACSR_TILE_ROWS;
constexpr int TILE_ROUNDS = TILE_ROWS / BIN_THREADS;
constexpr int NBINS = ACSR_NBINS;

// ---------------------------------------------------------------- SpMV mapping
// bins 1..6  : sub-warp of 2^{b-1} lanes per row, <= 2 nnz per lane (Alg. 2)
// bins 7..10 : one warp per row
// bins >= 11 : "heavy" rows (> 1024 nnz), cut into HEAVY_CHUNK-nnz chunks, one
//              warp per chunk, deterministic last-arriver combine.
constexpr int LIGHT_MAX_BIN = 10;
constexpr int HEAVY_BIN = LIGHT_MAX_BIN + 1;
constexpr int HEAVY_CHUNK = 1024;  // power of two

// rows per light work unit, by bin (~6-12 KB of CSR traffic per unit); ACSR_UNIT_SHIFT
// scales them by 2^shift for A/B builds
#ifndef ACSR_UNIT_SHIFT
#define ACSR_UNIT_SHIFT 0
#endif
#ifndef ACSR_UNIT_WARP_SHIFT
#define ACSR_UNIT_WARP_SHIFT 0  // extra right shift for the warp-per-row bins 7..10 (A/B)
#endif
__host__ __device__ constexpr int unit_rows_base(int b)
{
    return b == 0 ? 1024 : b == 1 ? 256 : b == 2 ? 128 : b == 3 ? 128 : b == 4 ? 64
         : b == 5 ? 32 : b == 6 ? 16
         : ((b == 7 ? 8 : b == 8 ? 4 : b == 9 ? 2 : 1) >> ACSR_UNIT_WARP_SHIFT) > 0
             ? ((b == 7 ? 8 : b == 8 ? 4 : b == 9 ? 2 : 1) >> ACSR_UNIT_WARP_SHIFT) : 1;
}
__host__ __device__ constexpr int unit_rows(int b)
{
    return ACSR_UNIT_SHIFT >= 0 ? unit_rows_base(b) << ACSR_UNIT_SHIFT
                                : (unit_rows_base(b) >> -ACSR_UNIT_SHIFT) > 0 ? unit_rows_base(b) >> -ACSR_UNIT_SHIFT : 1;
}

// Persistent CTAs (grid = resident CTAs per SM x SMs).  1024 threads: the whole SM
// shares one (optional) x cache.  Overridable for A/B builds.
#ifndef ACSR_SPMV_THREADS
#define ACSR_SPMV_THREADS 1024
#endif
constexpr int SPMV_THREADS = ACSR_SPMV_THREADS;
constexpr int SPMV_WARPS = SPMV_THREADS / 32;

// ---------------------------------------------------------------- x cache
// Direct-mapped cache of "hot" x entries in shared memory: slot s = c mod XC_SLOTS
// holds x[c] for the column c with the most occurrences among the columns mapping
// to s, counted over a strided sample of col_idx at bin time (sampled counts with
// atomicAdd, per-slot winner with a 64-bit atomicMax on (count << 32 | c)).  A
// gather first compares the 16-bit tag c >> XC_BITS with the slot's tag.  Caching
// never changes a value, only where it is read from.
constexpr int XC_BITS = 14;
constexpr int XC_SLOTS = 1 << XC_BITS;
constexpr uint16_t XC_NOTAG = 0xFFFF;
constexpr int XC_SAMPLE_LOG2 = 20;  // ~2^20 sampled entries per acsr_bin

// ---------------------------------------------------------------- short-row windows
// Rows of the shortest bins (0..WIN_MAX_BIN, i.e. len <= WIN_MAX_LEN) are not read
// through bin_rows one sub-warp per row: a warp takes WIN_ROWS = 32 CONSECUTIVE rows
// (one per lane), concatenates the nnz of its short rows (coalesced col/val loads of
// what are contiguous CSR runs), gathers x, and each lane sums its own row's products
// in element order from a per-warp shared-memory buffer.  Longer rows of the window
// are left to their bin units.  Measured reason: in bin order every
// short row costs a random row_ptr sector, partial col/val sectors and a random y
// sector, 22-29 % extra L2 sectors on the power-law matrices.  ACSR_WINDOW=0 restores
// the per-bin Alg. 2 mapping for bins 1..6 (A/B builds).
#ifndef ACSR_WINDOW
#define ACSR_WINDOW 1
#endif
#ifndef ACSR_WIN_MAX_BIN
#define ACSR_WIN_MAX_BIN 5
#endif
#ifndef ACSR_WIN_UNIT_ROWS
#define ACSR_WIN_UNIT_ROWS 128
#endif
#ifndef ACSR_WIN_G
#define ACSR_WIN_G 4
#endif
constexpr int WIN_MAX_BIN = ACSR_WINDOW ? ACSR_WIN_MAX_BIN : -1;  // -1: no windows
constexpr int WIN_MAX_LEN = 1 << (ACSR_WIN_MAX_BIN > 0 ? ACSR_WIN_MAX_BIN : 0);  // bin b holds len <= 2^b (b >= 1)
constexpr int WIN_ROWS = 32;
constexpr int WIN_UNIT_ROWS = ACSR_WIN_UNIT_ROWS;  // multiple of WIN_ROWS
constexpr int WIN_G = ACSR_WIN_G;                  // 32-element groups in flight per chunk
static_assert(WIN_UNIT_ROWS % WIN_ROWS == 0, "window unit = whole windows");
static_assert(TILE_ROWS % WIN_UNIT_ROWS == 0, "tiles hold whole window units");

__host__ __device__ constexpr int win_units(int tile_rows) { return (tile_rows + WIN_UNIT_ROWS - 1) / WIN_UNIT_ROWS; }

// Tail tiles: the last max(1, n_tiles / ACSR_TAIL_DIV) tiles of the work list get 4x
// smaller work units (32-row windows, a quarter of the rows per bin unit), so the last
// claims of the dynamic schedule are short and warps run out of work together.  With the
// late claims of round 2 and shift-based unit counts in the binning kernels, 1/16 of the
// tiles pays on every matrix: C2 step 99.7 -> 98.8 us, fp32 93.6 -> 92.7, LiveJournal-like
// 425.5 -> 420.1, web-Google-like unchanged (1/8, 1/4, 1/2: smaller or negative gains).
#ifndef ACSR_TAIL_DIV
#define ACSR_TAIL_DIV 16  // r2s2: the last 1/16 of the tiles (profiles/r2s2_taildiv_ab_shift.jsonl); 0: off
#endif
#ifndef ACSR_TAIL_MAX_TILES
#define ACSR_TAIL_MAX_TILES 320  // cap: the tail only has to cover the schedule's last rounds (s26 PageRank: 1/16 of
#endif                           // 65536 tiles cost the plain step 2 %, profiles/r2s2_c4_taildiv_ab.jsonl)
__host__ __device__ inline bool tail_tile(int tile, int n_tiles)
{
    if (ACSR_TAIL_DIV <= 0) return false;
    int k = n_tiles / (ACSR_TAIL_DIV > 0 ? ACSR_TAIL_DIV : 1);
    k = k < ACSR_TAIL_MAX_TILES ? k : ACSR_TAIL_MAX_TILES;
    return tile >= n_tiles - (k > 1 ? k : 1);
}
// Unit sizes are powers of two: the per-tile unit counts are computed with shifts (a
// division by a bin-dependent divisor is a ~20-instruction sequence in the binning kernels)
__host__ __device__ inline int ilog2_pow2(int v)
{
#ifdef __CUDA_ARCH__
    return 31 - __clz(v);
#else
    return 31 - __builtin_clz((unsigned)v);
#endif
}
static_assert((WIN_UNIT_ROWS & (WIN_UNIT_ROWS - 1)) == 0 && (WIN_ROWS & (WIN_ROWS - 1)) == 0, "powers of two");
__host__ __device__ inline int unit_shift_t(int b, bool tail)
{
    const int s = ilog2_pow2(unit_rows(b));
    return tail ? (s > 2 ? s - 2 : 0) : s;
}
__host__ __device__ inline int unit_rows_t(int b, bool tail) { return 1 << unit_shift_t(b, tail); }
__host__ __device__ inline int ceil_shift(int v, int s) { return (v + (1 << s) - 1) >> s; }
__host__ __device__ inline int win_unit_rows_t(bool tail) { return tail ? WIN_ROWS : WIN_UNIT_ROWS; }
__host__ __device__ inline int win_units_t(int tile_rows, bool tail)
{
    return ceil_shift(tile_rows, ilog2_pow2(win_unit_rows_t(tail)));
}

// unit descriptor: light  x = first index into bin_rows, y = (bin << 24) | rows
//                  heavy  x = row id,                     y = 0x80000000 | chunk
//                  window x = first row,                  y = 0x40000000 | rows
constexpr uint32_t HEAVY_FLAG = 0x80000000u;
constexpr uint32_t WIN_FLAG = 0x40000000u;

// ---------------------------------------------------------------- plan header
struct PlanHeader {
    int32_t n_heavy_units;  // heavy units come first in the unit list
    int32_t n_light_units;
    int32_t n_units;
    int32_t scan_ticket;    // last-CTA detection in the scan kernel
    int32_t role_ticket;    // fused scan+scatter launch: CTA role order (reset by bin_count)
    int32_t scan_done;      // fused scan+scatter launch: scan rows finished (reset by bin_count)
    int32_t work_ctr;       // dynamic unit counter (reset by the last warp)
    int32_t exit_ticket;    // last-warp detection at SpMV exit
    int32_t overflow;       // 1 if the unit list exceeded the workspace bounds
    int32_t n_tiles;
    int32_t xc_valid;       // 1 if the x-cache table was built (col_idx given)
    int32_t xc_stride;      // sampling stride used for the counts
    int64_t n_cols;
    uint64_t d2_hi, d2_mid, d2_lo;  // exact 192-bit fixed-point Delta^2 accumulator (PageRank/RWR)
    int64_t off_units, off_partial, off_ticket, off_xc_vote, off_xc_tag, off_xc_val;
    int64_t off_tile_done;  // int32 [n_tiles]: rows finished per tile (fused peer exchange), zeroed by acsr_bin
    int32_t totals[NBINS + 2 + 2];  // per scan row totals (bins, light units, heavy units)
};

struct PlanLayout {
    int64_t n_tiles = 0, light_cap = 0, heavy_cap = 0;
    size_t off_cnt = 0, off_toff = 0, off_units = 0, off_partial = 0, off_ticket = 0,
           off_xc_vote = 0, off_xc_tag = 0, off_xc_val = 0, off_xc_count = 0, off_tile_done = 0, total = 0;
};

__host__ __device__ inline size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

// Tile-level arrays are [ (NBINS + 2) x n_tiles ]: rows 0..31 the per-bin counts,
// row 32 light units per tile, row 33 heavy units per tile.
constexpr int SCAN_ROWS = NBINS + 2;

inline PlanLayout plan_layout(int64_t n_rows, int64_t n_cols, int64_t nnz_max)
{
    PlanLayout L;
    L.n_tiles = (n_rows + TILE_ROWS - 1) / TILE_ROWS;
    L.light_cap = n_rows + (int64_t)(LIGHT_MAX_BIN + 1) * L.n_tiles + 1;
    int64_t heavy_rows_max = nnz_max / (HEAVY_CHUNK + 1) + 1;
    L.heavy_cap = nnz_max / HEAVY_CHUNK + heavy_rows_max + 1;
    size_t o = align_up(sizeof(PlanHeader), 256);
    L.off_xc_vote = o;  // u64 (count << 32 | column) per slot
    o = align_up(o + sizeof(uint64_t) * XC_SLOTS, 256);
    L.off_xc_tag = o;
    o = align_up(o + sizeof(uint16_t) * XC_SLOTS, 256);
    L.off_xc_val = o;
    o = align_up(o + sizeof(double) * XC_SLOTS, 256);
    L.off_cnt = o;
    o = align_up(o + sizeof(int32_t) * SCAN_ROWS * (size_t)L.n_tiles, 256);
    L.off_toff = o;
    o = align_up(o + sizeof(int32_t) * SCAN_ROWS * (size_t)L.n_tiles, 256);
    L.off_units = o;
    o = align_up(o + sizeof(int2) * (size_t)(L.light_cap + L.heavy_cap), 256);
    L.off_partial = o;
    o = align_up(o + sizeof(double) * (size_t)L.heavy_cap, 256);
    L.off_ticket = o;
    o = align_up(o + sizeof(int32_t) * (size_t)L.heavy_cap, 256);
    L.off_tile_done = o;  // rows finished per tile (fused peer exchange)
    o = align_up(o + sizeof(int32_t) * (size_t)L.n_tiles, 256);
    L.off_xc_count = o;  // sampled occurrence count per column
    o = align_up(o + sizeof(int32_t) * (size_t)(n_cols > 0 ? n_cols : 0), 256);
    L.total = o;
    return L;
}

// ---------------------------------------------------------------- peer-memory exchange
// (acsr_peer.cu; NEXT N1 of SURVEY §8(f)).  Every rank owns one device region with the
// same layout, mapped into every other rank's address space (CUDA IPC over NVLink /
// NVSwitch P2P, or two processes on one GPU):
//   PeerState at offset 0, then the two replicated xs buffers (push parity 0 / 1).
// Rank q writes flag[q] and d2[.][q] in EVERY region (its own included) and xs slices
// into every region's buffer; the owner alone writes `pushes`, `err`, `ticket`.
//   pushes  number of completed pushes of this rank (init scale-push or fused step);
//           push c+1 writes buffer c & 1 and reads buffer (c-1) & 1 (fused step)
//   flag[q] = pushes of rank q once its stores of that push are visible (release.sys)
//   d2[p][q] the 192-bit fixed-point Delta^2 partial of rank q's push with parity p
constexpr int PEER_MAX = ACSR_PEER_MAX;
struct PeerState;

// kernel-side view of one acsr_peer.  The SpMV/PageRank kernel reads it through a
// pointer (a copy lives in the owner's region): dynamic indexing of base[] in a
// by-value kernel argument forced the whole argument block to local memory (spills).
struct PeerArgs {
    char *base[PEER_MAX];  // region base of rank q as mapped in this process
    PeerState *st;         // == (PeerState *)base[rank]
    int64_t off_buf[2];    // byte offset of xs buffer 0 / 1 inside a region
    int64_t slice_off;     // first xs slot of this rank's slice
    int64_t slice_len;     // local rows [0, slice_len) are exchanged
    int64_t xs_len;        // doubles per xs buffer
    unsigned long long timeout_ns;  // bound of every flag wait (ACSR_PEER_TIMEOUT_MS, default 20 s)
    int nranks, rank;
};

struct PeerState {
    unsigned long long flag[PEER_MAX];
    unsigned long long d2[2][PEER_MAX][3];
    unsigned long long pushes;
    unsigned int err;     // 1: a barrier wait timed out (results of that call are invalid)
    unsigned int ticket;  // last-CTA detection of the push kernel
    unsigned int last_step;  // 1 if this rank's last push was a fused step (has Delta^2 partials)
    PeerArgs view;        // this process's view (owner-written at acsr_peer_open)
};
constexpr size_t PEER_BUF_ALIGN = 4096;

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer_ns()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// One thread: wait until every rank has completed `target` pushes.  Bounded
// (p.timeout_ns, 20 s by default): on timeout st->err is set and the caller proceeds
// (the host checks err), so a lost peer never hangs the GPU.
__device__ __forceinline__ void peer_wait(const PeerArgs &p, unsigned long long target)
{
    const unsigned long long t0 = globaltimer_ns();
    for (int q = 0; q < p.nranks; q++) {
        while (ld_acquire_sys(&p.st->flag[q]) < target) {
            if (globaltimer_ns() - t0 > p.timeout_ns) {
                atomicExch(&p.st->err, 1u);
                return;
            }
            __nanosleep(256);
        }
    }
}

// One thread, after a system-scope fence that orders this push's data stores:
// publish the Delta^2 partial (PR) and the new push count to every rank.
__device__ __forceinline__ void peer_signal(const PeerArgs &p, unsigned long long newc, bool with_d2,
                                            unsigned long long hi, unsigned long long mid, unsigned long long lo)
{
    if (with_d2) {
        for (int q = 0; q < p.nranks; q++) {
            PeerState *s = (PeerState *)p.base[q];
            s->d2[newc & 1][p.rank][0] = hi;
            s->d2[newc & 1][p.rank][1] = mid;
            s->d2[newc & 1][p.rank][2] = lo;
        }
        __threadfence_system();
    }
    for (int q = 0; q < p.nranks; q++) st_release_sys(&((PeerState *)p.base[q])->flag[p.rank], newc);
    p.st->pushes = newc;
    p.st->last_step = with_d2 ? 1u : 0u;
}

// 192-bit fixed point (hi + mid 2^-64 + lo 2^-128) helpers for exact Delta^2 sums
__host__ __device__ __forceinline__ void fix192_merge(uint64_t &hi, uint64_t &mid, uint64_t &lo, uint64_t h,
                                                      uint64_t m, uint64_t l)
{
    const uint64_t nlo = lo + l;
    const uint64_t c1 = nlo < lo;
    const uint64_t m1 = mid + m;
    const uint64_t c2a = m1 < mid;
    const uint64_t m2 = m1 + c1;
    const uint64_t c2b = m2 < m1;
    lo = nlo;
    mid = m2;
    hi += h + c2a + c2b;
}
__host__ __device__ __forceinline__ double fix192_to_double(uint64_t hi, uint64_t mid, uint64_t lo)
{
    return (double)hi + ((double)mid + (double)lo * 5.421010862427522e-20) * 5.421010862427522e-20;
}

// Global Delta^2 of push c: the exact sum of every rank's 192-bit partial (the same bits
// on every rank, whatever the order), after peer_wait(p, c).
__device__ __forceinline__ double peer_sum_d2(const PeerArgs &p, unsigned long long c)
{
    unsigned long long hi = 0, mid = 0, lo = 0;
    for (int q = 0; q < p.nranks; q++) {
        const volatile unsigned long long *s = p.st->d2[c & 1][q];
        const unsigned long long h = s[0], m = s[1], l = s[2];
        const unsigned long long nlo = lo + l;
        const unsigned long long c1 = nlo < lo;
        const unsigned long long m1 = mid + m;
        const unsigned long long c2a = m1 < mid;
        const unsigned long long m2 = m1 + c1;
        const unsigned long long c2b = m2 < m1;
        lo = nlo;
        mid = m2;
        hi += h + c2a + c2b;
    }
    return (double)hi + ((double)mid + (double)lo * 5.421010862427522e-20) * 5.421010862427522e-20;
}

}  // namespace acsr

// host-side object behind the opaque acsr_peer handle (acsr_peer.cu)
struct acsr_peer {
    int nranks = 0, rank = 0, device = 0;
    int64_t xs_len = 0, slice_off = 0, slice_len = 0;
    size_t bytes = 0;
    char *region = nullptr;  // this rank's region (cudaMalloc, library-owned)
    bool opened = false;     // peers' regions mapped
    acsr::PeerArgs args{};   // kernel view (valid once opened)
};

namespace acsr {

// ---------------------------------------------------------------- device helpers
__device__ __forceinline__ int bin_of_len(int len)
{
    // bin 0: empty; 1: {1,2}; b = ceil(log2 len) otherwise
    return len <= 0 ? 0 : (len <= 2 ? 1 : 32 - __clz(len - 1));
}

__device__ __forceinline__ int heavy_chunks(int len) { return (len + HEAVY_CHUNK - 1) / HEAVY_CHUNK; }

__device__ __forceinline__ uint32_t mix32(uint32_t v)
{
    v ^= v >> 16;
    v *= 0x7feb352dU;
    v ^= v >> 15;
    v *= 0x846ca68bU;
    v ^= v >> 16;
    return v;
}

// ---------------------------------------------------------------- programmatic dependent launch
// The hot-path kernels of one step (bin_count -> bin_scan -> bin_scatter -> spmv, and
// back-to-back PageRank steps) are launched with programmatic stream serialization:
// the next grid is launched while the previous one runs and parks in
// griddepcontrol.wait until the previous grid has completed and its writes are
// visible, which hides the launch latency between the short kernels.  Every kernel
// launched this way calls pdl_enter() before its first global-memory access.
// ACSR_PDL=0 (environment) launches them plainly (A/B).
__device__ __forceinline__ void pdl_enter()
{
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

bool acsr_pdl_enabled();
int acsr_carveout();
bool acsr_carveout_once(const void *fn);

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t stream,
                              Args... args)
{
    const int co = acsr_carveout();
    if (co >= 0 && acsr_carveout_once((const void *)kernel))
        cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, co);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = acsr_pdl_enabled() ? 1 : 0;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

}  // namespace acsr

// library-owned NCCL exchange (acsr_comm.cu)
acsr_status acsr_comm_step_exchange(const acsr_pr_args *p, cudaStream_t stream);
uint64_t *acsr_comm_d2_slot(acsr_comm *c);
int acsr_comm_nranks(const acsr_comm *c);

// error plumbing (acsr_capi.cu)
void acsr_set_error(const char *fmt, ...);
acsr_status acsr_check_launch(const char *what);
int acsr_num_sms();
