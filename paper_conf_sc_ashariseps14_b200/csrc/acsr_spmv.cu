// acsr_spmv.cu -- bin-specific SpMV (Alg. 2) in ONE persistent launch, plus
// the fused PageRank step (Alg. 5).
//
// Work is cut by acsr_bin into warp-sized units (see acsr_internal.cuh):
//   heavy units   one HEAVY_CHUNK-nnz chunk of a row with > 1024 nnz; the last
//                 warp to finish a row (threadfence + atomic ticket) sums the
//                 chunk partials in chunk order (replaces the dynamic-parallelism
//                 parent/child kernels, Alg. 3/4).
//   light units   up to unit_rows(b) rows of one bin b <= 10 inside one 1024-row
//                 tile; bins 1..6 use a sub-warp of 2^{b-1} lanes per row and a
//                 width-2^{b-1} shuffle reduction (exactly Alg. 2 with reading Q6);
//                 bins 7..10 use a full warp per row; bin 0 writes +0.0 (Q2).
// Units are listed heavy-first, then tile by tile in row order.  Each warp starts
// on unit = its global warp id and then claims units from an atomic counter, so the
// GPU works on a narrow window of the row space (sectors shared by neighbouring rows
// of different bins are re-used from L2) and the tail is balanced.
//
// B200 specifics ("SpMV kernel"): the measured limiter of a plain
// gather-per-nonzero CSR SpMV on R-MAT graphs is the L1->L2 request rate of the
// random x gathers, not DRAM.  x therefore goes through a per-SM direct-mapped
// software cache of the hottest XC_SLOTS columns (tags + values in shared memory,
// filled once per call by TMA bulk copies from a compact array that a tiny
// pre-pass gathers) -- the B200 counterpart of binding x to texture memory.
//
// Every row is summed in an order that depends only on its length and address:
// y is deterministic run to run.  Accumulation is in double for both ACSR_F64 and
// ACSR_F32 (products of floats are exact in double).  The PageRank Delta^2 is
// accumulated in exact 128-bit fixed point (integer atomics), so it is
// deterministic too.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "acsr_internal.cuh"

#ifndef ACSR_BRANCHY_SUB
#define ACSR_BRANCHY_SUB 0  // 1: branchy element loads in the Alg. 2 sub-warp path (A/B builds)
#endif
#ifndef ACSR_NO_VEC
#define ACSR_NO_VEC 0  // 1: never use the 128-bit vector path (A/B builds)
#endif
#ifndef ACSR_PAIR_ROWS
#define ACSR_PAIR_ROWS 0  // 1: warp-per-row bins process two rows at a time (A/B builds)
#endif
#ifndef ACSR_MERGED_WARP_PATH
#define ACSR_MERGED_WARP_PATH 0  // 1: heavy + warp-per-row in one loop (A/B: PageRank s26 -0.8 %, SpMV C2/C3 +2-3 %)
#endif
#ifndef ACSR_WIN_LDS4
#define ACSR_WIN_LDS4 0  // 1: four shared loads in flight per add group (A/B: C3a +6 %, C2 +2 %, slower)
#endif
#ifndef ACSR_WIN_SEGSCAN
#define ACSR_WIN_SEGSCAN 0  // 1: segmented shuffle reduction per 32-element group (A/B r2f: C3a +24 %, C2 +4 %, LiveJournal-like +14 % -- SHFL shares the MIO path with the gathers)
#endif
#ifndef ACSR_WIN_SUM4
#define ACSR_WIN_SUM4 0  // 1: four accumulators by row offset mod 4 (A/B r2h: C3a 47.1 -> 49.2 us, C2 unchanged; kept off)
#endif
#ifndef ACSR_WIN_PREFETCH
#define ACSR_WIN_PREFETCH 0  // 1: prefetch the next window's row bounds (A/B: no gain on C3a, LiveJournal-like +5 %)
#endif
#ifndef ACSR_PF_UNIT
#define ACSR_PF_UNIT 0  // 1: L2 bulk prefetch of a unit's col/val runs at unit start (A/B)
#endif
#ifndef ACSR_PEER_TILE_PUSH
#define ACSR_PEER_TILE_PUSH 1  // 0: every finished row is stored to every peer at once (round-1 A/B)
#endif
#ifndef ACSR_DIAG
#define ACSR_DIAG 0  // diagnostics only (wrong results): 1 = no x gathers, 2 = no val loads, 3 = neither, 4 = no remote peer stores
#endif
#ifndef ACSR_PROF
#define ACSR_PROF 0  // diagnostics: per-mapping warp-cycle counters (acsr_debug_prof, A/B builds only)
#endif
#ifndef ACSR_CLAIM_GUIDED
#define ACSR_CLAIM_GUIDED 0  // > 0: guided batches of consecutive units per claim, k = left / (F * warps) (A/B)
#endif
#ifndef ACSR_GUIDED_AHEAD
#define ACSR_GUIDED_AHEAD 1  // guided batches: claim the next batch when the last unit of this one starts
#endif
#ifndef ACSR_WIN_LANE4
#define ACSR_WIN_LANE4 0  // 1: window chunk reduction by lanes owning 4 consecutive products + segmented suffix scan
#endif
#ifndef ACSR_DESC0
#define ACSR_DESC0 0  // first unit's descriptor with the plan header (host-known offset): 1 loaded, 2 L1 prefetch, 0 off
#endif
#ifndef ACSR_TIMELINE
#define ACSR_TIMELINE 0  // diagnostics: per-unit start/end cycles + SM id (acsr_debug_timeline, A/B builds only)
#endif
#ifndef ACSR_WIN_RPL
#define ACSR_WIN_RPL 1  // short-row window rows per lane (window = 32 * RPL consecutive rows)
#endif
#ifndef ACSR_WIN_DYN_SMEM
#define ACSR_WIN_DYN_SMEM (ACSR_WIN_G > 4 || ACSR_WIN_RPL > 1)  // window scratch in dynamic shared memory
#endif
#ifndef ACSR_PF_START_TILES
#define ACSR_PF_START_TILES 0  // > 0: L2 prefetch of the first tiles' CSR runs before the PDL wait only (A/B)
#endif
#ifndef ACSR_PF_TILES
#define ACSR_PF_TILES 0  // > 0: stream-ahead L2 prefetch of the CSR (col/val) this many 1024-row tiles ahead (A/B)
#endif
#ifndef ACSR_CLAIM_BATCH
#define ACSR_CLAIM_BATCH 0  // > 0: CTA-batched unit claims of this many units (A/B)
#endif
#ifndef ACSR_DESC_AHEAD
#define ACSR_DESC_AHEAD 0  // 1: claim two units ahead, load the next unit's descriptor during this one (A/B)
#endif
#ifndef ACSR_CLAIM_LATE
#define ACSR_CLAIM_LATE 1  // 1: claim the next unit when this one ends (r2af: C2 -3 %); 0: one prefetched claim; 2: prefetched until the last round
#endif
#ifndef ACSR_PR_STREAM_HINTS
#define ACSR_PR_STREAM_HINTS 0  // 1: evict-first hints for the PageRank epilogue's per-row vectors (A/B)
#endif
#ifndef ACSR_VEC_MIN
#define ACSR_VEC_MIN 1024  // rows (chunks) shorter than this use the lane-strided scalar path (r2ah: 512 -> 1024, C2 fp32 86.0 -> 84.0 us, others equal)
#endif


namespace acsr {

constexpr int WIN_TAB = 32 * ACSR_WIN_RPL;  // (row_begin, prefix) entries of a window's short rows

template <typename V>
struct SpmvArgs {
    const int32_t *__restrict__ rb;
    const int32_t *__restrict__ re;
    const int32_t *__restrict__ col;
    const V *__restrict__ val;
    const V *__restrict__ x;
    V *__restrict__ y;
    const int32_t *__restrict__ bin_rows;
    PlanHeader *hdr;
    // filled in-kernel from the plan header (offsets written by acsr_bin)
    const int2 *__restrict__ units;
    double *__restrict__ partial;
    int32_t *__restrict__ ticket;
    // shared-memory x cache (2^xc_bits slots)
    const uint16_t *xtag;
    const V *xval;
    int xc_bits;
    // 128-bit load phase: vector loads at element j need (j + vph) % 4 == 0; -1 = scalar only
    int vph;
    // PageRank epilogue
    const double *__restrict__ x_old;
    const int32_t *__restrict__ outdeg;
    double *__restrict__ x_new;
    double *__restrict__ xs_next;
    double damping, teleport;
    double *delta2;
    int64_t restart;
    double restart_weight;
    int32_t *ctrl;  // device-side convergence: [0] stop flag, [1] executed steps (nullable)
    double eps2;
    int64_t n_rows;  // rows of the call (NaN fill of an overflowed plan)
    uint64_t *d2_out;  // multi-GPU (acsr_comm): the last CTA writes this rank's exact 192-bit partial here
    int32_t *tile_done;  // fused peer exchange: rows finished per tile (plan workspace)
    int64_t x_prefetch;  // bytes of x to bulk-prefetch into L2 at entry (0: none)
    int64_t units_off;   // byte offset of the unit list in the plan (a function of n_rows alone), 0: unknown
    int64_t light_cap;   // unit-list entries guaranteed inside the plan (speculative first descriptor)
    // fused peer-memory exchange of xs_next (acsr_pagerank_step_peer; peer.nranks == 0: off)
    const PeerArgs *peer;  // device copy (PeerState::view) or NULL
    // set in-kernel from *peer (registers + a shared copy of the region bases), so the
    // per-row epilogue does not re-load the peer view
    char *const *pbase;    // shared: region base of every rank
    char *pself;           // region base of this rank
    int64_t peer_next;     // byte offset of the buffer this step pushes into
    int64_t peer_off;      // slice_off
    int peer_len, peer_n;  // slice_len (< 2^31, local rows), nranks
    int peer_rank;
};

// ----------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar)
{
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase)
{
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(phase)
            : "memory");
    }
}

// 192-bit fixed point (value = hi + mid * 2^-64 + lo * 2^-128) for exact,
// order-independent sums of non-negative doubles below 2^64: Delta^2 of any step is
// deterministic under dynamic scheduling.  Each term is split exactly (53-bit mantissa)
// and truncated below 2^-128.
struct Fix192 {
    uint64_t hi, mid, lo;
    int fin, ftile;  // fused peer exchange: rows this lane finished in the current unit, their tile
};

__device__ __forceinline__ void fix_merge(Fix192 &a, uint64_t hi, uint64_t mid, uint64_t lo)
{
    const uint64_t nlo = a.lo + lo;
    const uint64_t c1 = nlo < a.lo ? 1u : 0u;
    const uint64_t m1 = a.mid + mid;
    const uint64_t c2a = m1 < a.mid ? 1u : 0u;
    const uint64_t m2 = m1 + c1;
    const uint64_t c2b = m2 < m1 ? 1u : 0u;
    a.lo = nlo;
    a.mid = m2;
    a.hi += hi + c2a + c2b;
}

__device__ __forceinline__ void fix_add(Fix192 &a, double d)
{
    if (!(d > 0.0)) return;
    if (d >= 18446744073709549568.0) d = 18446744073709549568.0;  // < 2^64 (saturate)
    const double hf = floor(d);
    const double r1 = (d - hf) * 18446744073709551616.0;  // exact: * 2^64
    const double mf = floor(r1);
    const double r2 = (r1 - mf) * 18446744073709551616.0;
    fix_merge(a, (uint64_t)hf, (uint64_t)mf, (uint64_t)floor(r2));
}

// ----------------------------------------------------------------- load flavours
// Streamed CSR arrays (col, val) and the gathered x use separate cache policies.
// Compile-time choice (ACSR_STREAM_LD / ACSR_X_LD) so variants can be A/B-measured:
//   ACSR_STREAM_LD 0: ld.global.cs (evict-first)   1: ld.global.nc.L1::no_allocate
//                  2: ld.global.nc.L1::no_allocate + L2 evict_first cache policy
//   ACSR_X_LD      0: ld.global.nc                 1: ld.global.nc.L1::evict_last
//                  2: ld.global.nc + L2 evict_last cache policy (createpolicy)
#ifndef ACSR_STREAM_LD
#define ACSR_STREAM_LD 0
#endif
#ifndef ACSR_X_LD
#define ACSR_X_LD 0
#endif

__device__ __forceinline__ uint64_t pol_evict_first()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_evict_last()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}

__device__ __forceinline__ int lds_i(const int *p)
{
#if ACSR_STREAM_LD == 2
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
#else
    return __ldcs(p);
#endif
}
__device__ __forceinline__ double lds_d(const double *p)
{
#if ACSR_STREAM_LD == 2
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    double v;
    asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
#else
    return __ldcs(p);
#endif
}
__device__ __forceinline__ float lds_f(const float *p)
{
#if ACSR_STREAM_LD == 2
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
#else
    return __ldcs(p);
#endif
}
__device__ __forceinline__ int4 lds_i4(const int *p)
{
#if ACSR_STREAM_LD == 2
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
#else
    return __ldcs(reinterpret_cast<const int4 *>(p));
#endif
}
__device__ __forceinline__ double2 lds_d2(const double *p)
{
#if ACSR_DIAG == 2 || ACSR_DIAG == 3
    return make_double2(1.0, 1.0 + (double)((uintptr_t)p & 1));
#endif
#if ACSR_STREAM_LD == 2
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
#else
    return __ldcs(reinterpret_cast<const double2 *>(p));
#endif
}
__device__ __forceinline__ float4 lds_f4(const float *p)
{
#if ACSR_DIAG == 2 || ACSR_DIAG == 3
    return make_float4(1.f, 1.f, 1.f, 1.f + (float)((uintptr_t)p & 1));
#endif
#if ACSR_STREAM_LD == 2
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol_evict_first()));
    return v;
#elif ACSR_STREAM_LD == 1
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
#else
    return __ldcs(reinterpret_cast<const float4 *>(p));
#endif
}
#if ACSR_DIAG == 2 || ACSR_DIAG == 3
__device__ __forceinline__ double lds_v(const double *p) { return 1.0 + (double)((uintptr_t)p & 1); }
__device__ __forceinline__ double lds_v(const float *p) { return 1.0 + (double)((uintptr_t)p & 1); }
#else
__device__ __forceinline__ double lds_v(const double *p) { return lds_d(p); }
__device__ __forceinline__ double lds_v(const float *p) { return (double)lds_f(p); }
#endif

__device__ __forceinline__ double ldx(const double *p)
{
#if ACSR_DIAG == 1 || ACSR_DIAG == 3
    return 1.0 + (double)((uintptr_t)p & 1);  // no load (the address still depends on col)
#endif
#if ACSR_X_LD == 2
    double v;
    asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol_evict_last()));
    return v;
#elif ACSR_X_LD == 1
    double v;
    asm volatile("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
#else
    return __ldg(p);
#endif
}
__device__ __forceinline__ double ldx(const float *p)
{
#if ACSR_DIAG == 1 || ACSR_DIAG == 3
    return 1.0 + (double)((uintptr_t)p & 1);
#endif
#if ACSR_X_LD == 2
    float v;
    asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol_evict_last()));
    return (double)v;
#elif ACSR_X_LD == 1
    float v;
    asm volatile("ld.global.nc.L1::evict_last.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return (double)v;
#else
    return (double)__ldg(p);
#endif
}

__device__ __forceinline__ bool cb_valid(int cb, int T) { return cb < T; }

#if ACSR_PROF
// [0] window units  [1] light_sub units  [2] light_warp units  [3] heavy units  [4] empty units
// [5] window: row-bounds wait  [6] window: chunk loads + gathers  [7] window: in-order sums
// [8] kernel entry -> first unit  [9] last unit -> exit  [10..14] unit counts by type
// [15] launches
__device__ unsigned long long g_prof[16];
#define PROF_ADD(i, v) atomicAdd(&g_prof[i], (unsigned long long)(v))
#endif

#if ACSR_TIMELINE
// per unit u < TL_MAX: {start, end} in SM cycles since the CTA's entry, packed with the SM id
// (bits 48..55) and the unit kind (bits 56..59); g_tl_cta[b] = {globaltimer at CTA entry, clock64
// at entry, globaltimer at the CTA's exit}
constexpr int TL_MAX = 1 << 16;
__device__ unsigned long long g_tl[TL_MAX][2];
__device__ unsigned long long g_tl_cta[1024][3];
__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned smid()
{
    unsigned r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}
#endif

// xs' slice entry -> every OTHER rank's replicated buffer (byte offset o in each region)
__device__ __noinline__ void peer_store(char *const *pbase, int nranks, int self, int64_t o, double v)
{
    for (int q = 0; q < nranks; q++)
        if (q != self) *(double *)(pbase[q] + o) = v;
}

template <typename V, bool HAS_VAL, bool HAS_END, bool PR, bool XC, bool PEER = false>
struct Kern {
    using A = SpmvArgs<V>;

    static __device__ __forceinline__ void row_bounds(const A &a, int r, int &beg, int &end)
    {
        beg = __ldg(a.rb + r);
        end = HAS_END ? __ldg(a.re + r) : __ldg(a.rb + r + 1);
    }

    static __device__ __forceinline__ double gx(const A &a, int c)
    {
        if (XC) {
            const uint32_t s = (uint32_t)c & ((1u << a.xc_bits) - 1u);
            if (a.xtag[s] == (uint16_t)((uint32_t)c >> a.xc_bits)) return (double)a.xval[s];
        }
        return ldx(a.x + c);
    }

    static __device__ __forceinline__ double prod(const A &a, int k)
    {
        const int c = lds_i(a.col + k);
        const double xv = gx(a, c);
        if (HAS_VAL) return lds_v(a.val + k) * xv;
        return xv;
    }

    static __device__ __forceinline__ double fmac(const A &a, int k, double acc)
    {
        const int c = lds_i(a.col + k);
        const double xv = gx(a, c);
        if (HAS_VAL) return fma(lds_v(a.val + k), xv, acc);
        return acc + xv;
    }

    // cp.async.bulk.prefetch.L2 of the element range [kb, ke) of col (and val): the rows
    // of a unit are processed one after another, so the later rows' CSR runs come from L2
    // instead of DRAM (ACSR_PF_UNIT)
    static __device__ __forceinline__ void pf_bytes(const void *p, int64_t bytes)
    {
        uintptr_t b = (uintptr_t)p & ~(uintptr_t)15;
        const uintptr_t e = ((uintptr_t)p + (uintptr_t)bytes + 15) & ~(uintptr_t)15;
        while (b < e) {
            const uint32_t sz = (uint32_t)(e - b < 32768 ? e - b : 32768);
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(b), "r"(sz) : "memory");
            b += sz;
        }
    }
    static __device__ __forceinline__ void pf_range(const A &a, int kb, int ke)
    {
        if (ke <= kb) return;
        pf_bytes(a.col + kb, 4 * (int64_t)(ke - kb));
        if (HAS_VAL) pf_bytes(a.val + kb, (int64_t)sizeof(V) * (ke - kb));
    }

    // write the row result (or the PageRank epilogue for local row r)
    static __device__ __forceinline__ void finish(const A &a, int r, double s, Fix192 &d2)
    {
        if (PR) {
            const double xn = a.teleport + a.damping * s + (r == a.restart ? a.restart_weight : 0.0);
#if ACSR_PR_STREAM_HINTS
            // x_new / x_old / outdeg are touched once per step: streaming (evict-first) so they
            // do not push the hot xs lines out of L2; xs_next keeps the default policy (the next
            // step gathers it)
            __stcs(a.x_new + r, xn);
            const int od = __ldcs(a.outdeg + r);
#else
            a.x_new[r] = xn;
            const int od = __ldg(a.outdeg + r);
#endif
            const double xs = od > 0 ? xn / (double)od : 0.0;
            if (a.xs_next) a.xs_next[r] = xs;  // NULL: peer exchange only
            // the exchange, fused: store the slice entry straight into every rank's
            // replicated xs (NVLink P2P stores; window rows give coalesced 256-B runs).
            // The remote loop is out of line: inlined at every finish() site it cost
            // I-cache misses (ncu no_instruction stalls 0.9 -> 3.3 per issue, +13 %).
            if (PEER && r < a.peer_len) {
                const int64_t o = a.peer_next + 8 * (a.peer_off + r);
                *(double *)(a.pself + o) = xs;  // own replicated buffer: inline
                if (!ACSR_PEER_TILE_PUSH && ACSR_DIAG != 4 && a.peer_n > 1)
                    peer_store(a.pbase, a.peer_n, a.peer_rank, o, xs);
            }
            if (PEER) {  // per-tile completion count (peer_tile_done)
                d2.fin++;
                d2.ftile = r / TILE_ROWS;
            }
#if ACSR_PR_STREAM_HINTS
            const double diff = xn - __ldcs(a.x_old + r);
#else
            const double diff = xn - __ldg(a.x_old + r);
#endif
            fix_add(d2, diff * diff);
        } else {
            a.y[r] = (V)s;
        }
    }

    // bins 1..6: W = 2^{b-1} lanes per row, each lane <= 2 elements (Alg. 2)
    template <int W>
    static __device__ __forceinline__ void light_sub(const A &a, int start, int cnt, int lane, Fix192 &d2)
    {
        constexpr int RPP = 32 / W;           // rows per pass
        constexpr int U = (W >= 16) ? 2 : 4;  // passes in flight
        const int sub = lane / W, li = lane % W;
        for (int i0 = 0; i0 < cnt; i0 += RPP * U) {
            int r[U], beg[U], end[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int i = i0 + u * RPP + sub;
                r[u] = i < cnt ? __ldg(a.bin_rows + start + i) : -1;
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
                if (r[u] >= 0) row_bounds(a, r[u], beg[u], end[u]);
                else beg[u] = end[u] = 0;
            }
            double acc[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int k0 = beg[u] + li, k1 = k0 + W;
#if ACSR_BRANCHY_SUB
                double sacc = 0.0;
                if (k0 < end[u]) sacc = prod(a, k0);
                if (k1 < end[u]) sacc += prod(a, k1);
                acc[u] = sacc;
#else
                acc[u] = fmacp(a, k0 < end[u], k0, 0.0);
                acc[u] = fmacp(a, k1 < end[u], k1, acc[u]);
#endif
            }
#pragma unroll
            for (int u = 0; u < U; u++) {
#pragma unroll
                for (int o = W / 2; o > 0; o >>= 1) acc[u] += __shfl_down_sync(0xffffffffu, acc[u], o, W);
                if (li == 0 && r[u] >= 0) finish(a, r[u], acc[u], d2);
            }
        }
    }

    static __device__ __forceinline__ double warp_sum(double v)
    {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        return v;
    }

    // predicated gather: p false => 0 without touching memory
    static __device__ __forceinline__ double gxp(const A &a, bool p, int c)
    {
        double v = 0.0;
        if (XC) {
            const uint32_t s = (uint32_t)c & ((1u << a.xc_bits) - 1u);
            const bool hit = p && a.xtag[s] == (uint16_t)((uint32_t)c >> a.xc_bits);
            if (hit) v = (double)a.xval[s];
            if (p && !hit) v = ldx(a.x + c);
        } else {
            if (p) v = ldx(a.x + c);
        }
        return v;
    }

    // masked scalar element: contributes val[k] * x[col[k]] only when p
    static __device__ __forceinline__ double fmacp(const A &a, bool p, int k, double acc)
    {
        const int c = p ? lds_i(a.col + k) : 0;
        const double xv = gxp(a, p, c);
        if (HAS_VAL) {
            const double v = p ? lds_v(a.val + k) : 0.0;
            return fma(v, xv, acc);
        }
        return acc + xv;
    }

    // lane-strided dot over [kb, ke).
    // Vector path (rows >= 64 nnz): a scalar head of <= 3 elements up to the first index
    // j_a with (j_a + vph) % 4 == 0, then groups of 128 consecutive elements with one
    // 128-bit col load (int4) and 128-bit val loads per lane, TWO groups per iteration
    // issued back to back (8 gathers in flight per lane, no branches in the body), then
    // a lane-strided masked tail.  Element t of a lane's 4-vector always feeds
    // accumulator t: the summation order depends only on (kb, ke, vph).
    static __device__ __forceinline__ double strided_dot(const A &a, int kb, int ke, int lane)
    {
        double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
        int k;
        if (a.vph >= 0 && ke - kb >= ACSR_VEC_MIN) {
            const int ja = ((kb + a.vph + 3) & ~3) - a.vph;  // first aligned index >= kb
            s0 = fmacp(a, lane < ja - kb, kb + lane, s0);
            int j = ja;
            for (; j + 256 <= ke; j += 256) {
                const int e0 = j + 4 * lane, e1 = e0 + 128;
                const int4 c0 = lds_i4(a.col + e0);
                const int4 c1 = lds_i4(a.col + e1);
                double v[8];
                if (HAS_VAL) {
                    if (sizeof(V) == 8) {
                        const double2 p0 = lds_d2((const double *)(a.val + e0));
                        const double2 p1 = lds_d2((const double *)(a.val + e0 + 2));
                        const double2 p2 = lds_d2((const double *)(a.val + e1));
                        const double2 p3 = lds_d2((const double *)(a.val + e1 + 2));
                        v[0] = p0.x; v[1] = p0.y; v[2] = p1.x; v[3] = p1.y;
                        v[4] = p2.x; v[5] = p2.y; v[6] = p3.x; v[7] = p3.y;
                    } else {
                        const float4 p0 = lds_f4((const float *)(a.val + e0));
                        const float4 p1 = lds_f4((const float *)(a.val + e1));
                        v[0] = p0.x; v[1] = p0.y; v[2] = p0.z; v[3] = p0.w;
                        v[4] = p1.x; v[5] = p1.y; v[6] = p1.z; v[7] = p1.w;
                    }
                }
                const double x0 = gx(a, c0.x), x1 = gx(a, c0.y), x2 = gx(a, c0.z), x3 = gx(a, c0.w);
                const double x4 = gx(a, c1.x), x5 = gx(a, c1.y), x6 = gx(a, c1.z), x7 = gx(a, c1.w);
                if (HAS_VAL) {
                    s0 = fma(v[0], x0, s0); s1 = fma(v[1], x1, s1); s2 = fma(v[2], x2, s2); s3 = fma(v[3], x3, s3);
                    s0 = fma(v[4], x4, s0); s1 = fma(v[5], x5, s1); s2 = fma(v[6], x6, s2); s3 = fma(v[7], x7, s3);
                } else {
                    s0 += x0; s1 += x1; s2 += x2; s3 += x3;
                    s0 += x4; s1 += x5; s2 += x6; s3 += x7;
                }
            }
            k = j + lane;  // tail (< 256 elements), lane-strided, masked, 4 in flight
        } else {
            k = kb + lane;
        }
        for (; k < ke; k += 128) {
            s0 = fmacp(a, true, k, s0);
            s1 = fmacp(a, k + 32 < ke, k + 32, s1);
            s2 = fmacp(a, k + 64 < ke, k + 64, s2);
            s3 = fmacp(a, k + 96 < ke, k + 96, s3);
        }
        return (s0 + s1) + (s2 + s3);
    }

    // bins 7..10: a warp per row
    static __device__ __forceinline__ void light_warp(const A &a, int start, int cnt, int lane, Fix192 &d2)
    {
        const int myr = lane < cnt ? __ldg(a.bin_rows + start + lane) : 0;
        int mb = 0, me = 0;
        if (lane < cnt) row_bounds(a, myr, mb, me);
        if (ACSR_PF_UNIT && lane > 0 && lane < cnt) pf_range(a, mb, me);  // rows 1.. of the unit
#if ACSR_PAIR_ROWS
        // two rows in flight: element k of a row feeds accumulator (k mod 64) < 32 ? p : q,
        // whether or not the row has a partner -> per-row order independent of pairing
        for (int i = 0; i < cnt; i += 2) {
            const bool has1 = i + 1 < cnt;
            const int r0 = __shfl_sync(0xffffffffu, myr, i);
            const int b0 = __shfl_sync(0xffffffffu, mb, i);
            const int l0 = __shfl_sync(0xffffffffu, me, i) - b0;
            const int r1 = __shfl_sync(0xffffffffu, myr, has1 ? i + 1 : i);
            const int b1 = __shfl_sync(0xffffffffu, mb, has1 ? i + 1 : i);
            const int l1 = has1 ? __shfl_sync(0xffffffffu, me, i + 1) - b1 : 0;
            double p0 = 0.0, q0 = 0.0, p1 = 0.0, q1 = 0.0;
            const int L = max(l0, l1);
            for (int k = lane; k < L; k += 64) {
                p0 = fmacp(a, k < l0, b0 + k, p0);
                q0 = fmacp(a, k + 32 < l0, b0 + k + 32, q0);
                p1 = fmacp(a, k < l1, b1 + k, p1);
                q1 = fmacp(a, k + 32 < l1, b1 + k + 32, q1);
            }
            const double s0 = warp_sum(p0 + q0);
            const double s1 = warp_sum(p1 + q1);
            if (lane == 0) {
                finish(a, r0, s0, d2);
                if (has1) finish(a, r1, s1, d2);
            }
        }
        return;
#endif
        for (int i = 0; i < cnt; i++) {
            const int r = __shfl_sync(0xffffffffu, myr, i);
            const int beg = __shfl_sync(0xffffffffu, mb, i);
            const int end = __shfl_sync(0xffffffffu, me, i);
            const double s = warp_sum(strided_dot(a, beg, end, lane));
            if (lane == 0) finish(a, r, s, d2);
        }
    }

    // masked product: val[k] * x[col[k]] when p, else 0 (no memory touched)
    static __device__ __forceinline__ double prodp(const A &a, bool p, int k)
    {
        const int c = p ? lds_i(a.col + k) : 0;
        const double xv = gxp(a, p, c);
        if (HAS_VAL) return (p ? lds_v(a.val + k) : 0.0) * xv;
        return xv;
    }

    // Short-row windows (acsr_internal.cuh): rows r0 .. r0+nrows-1, 32 per pass, lane i
    // owns row r0 + w + i.  The nnz of the window's short rows (len <= WIN_MAX_LEN) are
    // concatenated in row order; element t of the concatenation is loaded by lane
    // t mod 32 (coalesced over the CSR runs), its row found from the head bitmask of the
    // 32-element group and a per-warp (beg, pre) table of the non-empty short rows.
    // Products go to a per-warp shared buffer; each lane then adds ITS row's products in
    // element order, so a row's sum depends only on the row (as in every other mapping).
#if ACSR_WIN_RPL > 1
    // Wide short-row windows (ACSR_WIN_RPL rows per lane): the same mapping as window()
    // below, but a warp concatenates 32 * RPL consecutive rows at once (row i of the window
    // = lane + 32 j, j < RPL), so one row-bounds round trip and each chunk of 32 * WIN_G
    // elements serve RPL times more rows (short-row matrices: more elements per dependent
    // memory round trip).  Each lane sums its RPL rows' products in element order.
    static __device__ __forceinline__ void window(const A &a, int r0, int nrows, int lane, Fix192 &d2,
                                                  double *buf, int2 *tab)
    {
        constexpr unsigned FULL = 0xffffffffu;
        constexpr int RPL = ACSR_WIN_RPL, WR = 32 * RPL, CH = 32 * WIN_G;
        const unsigned lt = (1u << lane) - 1u;
        const unsigned le = 0xffffffffu >> (31 - lane);
        for (int w = 0; w < nrows; w += WR) {
            int beg[RPL], l[RPL], pre[RPL];
            bool mine[RPL];
#pragma unroll
            for (int j = 0; j < RPL; j++) {
                const int i = w + j * 32 + lane;
                int b = 0, e = 0;
                if (i < nrows) row_bounds(a, r0 + i, b, e);
                beg[j] = b;
                mine[j] = i < nrows && e - b <= WIN_MAX_LEN;
                l[j] = mine[j] ? e - b : 0;
            }
            int base = 0, nbase = 0;
#pragma unroll
            for (int j = 0; j < RPL; j++) {
                int incl = l[j];
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const int t = __shfl_up_sync(FULL, incl, d);
                    if (lane >= d) incl += t;
                }
                pre[j] = base + incl - l[j];
                const unsigned ne = __ballot_sync(FULL, l[j] > 0);
                if (l[j] > 0) tab[nbase + __popc(ne & lt)] = make_int2(beg[j], pre[j]);
                base += __shfl_sync(FULL, incl, 31);
                nbase += __popc(ne);
            }
            const int T = base;
            __syncwarp();
            double acc[RPL];
#pragma unroll
            for (int j = 0; j < RPL; j++) acc[j] = 0.0;
            for (int t0 = 0; t0 < T; t0 += CH) {
                double p[WIN_G];
#pragma unroll
                for (int g = 0; g < WIN_G; g++) {
                    const int cb = t0 + 32 * g;
                    unsigned hb = 0;
                    int qc = 0;
#pragma unroll
                    for (int j = 0; j < RPL; j++) {
                        const bool hd = l[j] > 0 && pre[j] >= cb && pre[j] < cb + 32;
                        hb |= hd ? 1u << (pre[j] - cb) : 0u;
                        qc += __popc(__ballot_sync(FULL, l[j] > 0 && pre[j] < cb));
                    }
                    const unsigned H = __reduce_or_sync(FULL, hb);
                    const bool v = cb + lane < T;
                    const int t = v ? cb + lane : T - 1;
                    const int2 bp = tab[qc + __popc(H & le) - 1];
                    const int k = bp.x + (t - bp.y);
                    const int c = lds_i(a.col + k);
                    const double xv = gx(a, c);
                    const double pv = HAS_VAL ? lds_v(a.val + k) * xv : xv;
                    p[g] = v ? pv : 0.0;
                }
#pragma unroll
                for (int g = 0; g < WIN_G; g++) buf[32 * g + lane] = p[g];
                __syncwarp();
#pragma unroll
                for (int j = 0; j < RPL; j++) {
                    if (l[j] > 0) {
                        const int i1 = min(pre[j] + l[j], t0 + CH) - t0;
                        for (int i = max(pre[j], t0) - t0; i < i1; i++) acc[j] += buf[i];
                    }
                }
                __syncwarp();
            }
#pragma unroll
            for (int j = 0; j < RPL; j++)
                if (mine[j]) finish(a, r0 + w + j * 32 + lane, acc[j], d2);
            __syncwarp();  // tab / buf reused by the next window
        }
    }
#else
    static __device__ __forceinline__ void window(const A &a, int r0, int nrows, int lane, Fix192 &d2,
                                                  double *buf, int2 *tab)
    {
        constexpr unsigned FULL = 0xffffffffu;
        const unsigned lt = (1u << lane) - 1u;
        const unsigned le = 0xffffffffu >> (31 - lane);
        if (ACSR_PF_UNIT && nrows > WIN_ROWS && lane == 0) {
            // the unit's rows are consecutive: one contiguous CSR run (windows 2.. of the unit)
            const int kb = __ldg(a.rb + r0 + WIN_ROWS);
            const int ke = HAS_END ? __ldg(a.re + r0 + nrows - 1) : __ldg(a.rb + r0 + nrows);
            pf_range(a, kb, ke);
        }
#if ACSR_WIN_PREFETCH
        // the next window's row bounds are loaded while this window runs (one dependent
        // DRAM round trip less per window on short-row matrices)
        int nbeg = 0, nend = 0;
        if (lane < nrows) row_bounds(a, r0 + lane, nbeg, nend);
#endif
        for (int w = 0; w < nrows; w += WIN_ROWS) {
            const int r = r0 + w + lane;
            const bool in = w + lane < nrows;
            int beg = 0, end = 0;
#if ACSR_WIN_PREFETCH
            beg = nbeg;
            end = nend;
            nbeg = nend = 0;
            if (w + WIN_ROWS + lane < nrows) row_bounds(a, r + WIN_ROWS, nbeg, nend);
#else
            if (in) row_bounds(a, r, beg, end);
#endif
#if ACSR_PROF
            long long pt0 = clock64();
#endif
            const int len = end - beg;
#if ACSR_PROF
            {
                const int lsync = __shfl_sync(FULL, len, 0);  // forces the wait here
                if (lane == 0 && lsync >= 0) PROF_ADD(5, clock64() - pt0);
                pt0 = clock64();
            }
#endif
            const bool mine = in && len <= WIN_MAX_LEN;
            const int l = mine ? len : 0;
            int incl = l;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const int t = __shfl_up_sync(FULL, incl, d);
                if (lane >= d) incl += t;
            }
            const int pre = incl - l;
            const int T = __shfl_sync(FULL, incl, 31);
            const unsigned ne = __ballot_sync(FULL, l > 0);
            if (l > 0) tab[__popc(ne & lt)] = make_int2(beg, pre);
#if ACSR_WIN_SEGSCAN
            buf[lane] = 0.0;  // per-row partial sums (tab index)
#endif
            __syncwarp();
            double acc = 0.0;
#if ACSR_WIN_SUM4
            double a1 = 0.0, a2 = 0.0, a3 = 0.0;
#endif
#if ACSR_WIN_LANE4
            double pend_s = 0.0;  // the row left open at the end of the previous chunk: partial sum,
            int pend_rj = -1;     // and its table index (-1: none)
#endif
            for (int t0 = 0; t0 < T; t0 += 32 * WIN_G) {
                double p[WIN_G];
#if ACSR_WIN_SEGSCAN
                int rjg[WIN_G];
#endif
#if ACSR_WIN_LANE4
                unsigned Hs[WIN_G];
                int Q0 = 0;
#endif
#pragma unroll
                for (int g = 0; g < WIN_G; g++) {
                    const int cb = t0 + 32 * g;
                    const bool hd = l > 0 && pre >= cb && pre < cb + 32;
                    const unsigned H = __reduce_or_sync(FULL, hd ? 1u << (pre - cb) : 0u);
                    const int q0 = __popc(__ballot_sync(FULL, l > 0 && pre < cb));
#if ACSR_WIN_LANE4
                    Hs[g] = H;
                    if (g == 0) Q0 = q0;
#endif
                    // element t, clamped to the last one (T-1) past the end so that every
                    // lane loads from a valid address: no branches, all WIN_G groups'
                    // loads are issued back to back (the f32 build serialised them when
                    // the loads sat behind a branch).  No row starts at or past T, so the
                    // row found for a clamped lane is the last non-empty row, which holds T-1.
                    const bool v = cb + lane < T;
                    const int t = v ? cb + lane : T - 1;
                    const int rj = q0 + __popc(H & le) - 1;  // the element's row (tab index)
                    const int2 bp = tab[rj];
                    const int k = bp.x + (t - bp.y);
                    const int c = lds_i(a.col + k);
                    const double xv = gx(a, c);
                    const double pv = HAS_VAL ? lds_v(a.val + k) * xv : xv;
                    p[g] = v ? pv : 0.0;
#if ACSR_WIN_SEGSCAN
                    rjg[g] = rj;
#endif
                }
#if ACSR_WIN_SEGSCAN
                // segmented reduction of each 32-element group by shuffles (rows are
                // contiguous lane runs, the row index rj is non-decreasing across lanes):
                // after the inclusive segmented scan the last lane of each run holds the
                // run's sum and adds it to the row's partial in shared memory (groups in
                // order -> deterministic for a given window)
#pragma unroll
                for (int g = 0; g < WIN_G; g++) {
                    double sv = p[g];
                    const int rj = rjg[g];
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
                        const double o = __shfl_up_sync(FULL, sv, d);
                        const int orj = __shfl_up_sync(FULL, rj, d);
                        if (lane >= d && orj == rj) sv += o;
                    }
                    const int nrj = __shfl_down_sync(FULL, rj, 1);
                    if (cb_valid(t0 + 32 * g, T) && (lane == 31 || nrj != rj)) buf[rj] += sv;
                    __syncwarp();
                }
#elif ACSR_WIN_LANE4
                static_assert(WIN_G == 4, "lane-4 reduction: 128-element chunks, 4 consecutive products per lane");
                // Lane i takes the chunk's products 4i .. 4i+3 (two 16-byte shared loads, no bank
                // conflicts) and sums them per row in element order in registers: the row heads
                // among its 4 elements are bits 4(i mod 8) .. +3 of group i/8's head mask.  A row
                // whose elements spill into the following lanes gets their leading parts through
                // one segmented suffix scan over the lanes (5 shuffle levels per 128 elements,
                // instead of a per-lane loop of shared loads over the longest row).  Finished row
                // sums go to the row's table slot (tab is not read for a finished row again); the
                // row open at the chunk's end is completed by the next chunk's leading elements.
#pragma unroll
                for (int g = 0; g < WIN_G; g++) buf[32 * g + lane] = p[g];
                __syncwarp();
                {
                    const double2 qa = *(const double2 *)(buf + 4 * lane);
                    const double2 qb = *(const double2 *)(buf + 4 * lane + 2);
                    const double q[4] = {qa.x, qa.y, qb.x, qb.y};
                    const int gs = lane >> 3;
                    const unsigned Hl = gs == 0 ? Hs[0] : gs == 1 ? Hs[1] : gs == 2 ? Hs[2] : Hs[3];
                    const int sh = 4 * (lane & 7);
                    const unsigned hb = (Hl >> sh) & 0xFu;
                    int hi = Q0 + __popc(Hl & ((1u << sh) - 1u)) + (gs > 0 ? __popc(Hs[0]) : 0) +
                             (gs > 1 ? __popc(Hs[1]) : 0) + (gs > 2 ? __popc(Hs[2]) : 0);
                    double *res = (double *)tab;
#if ACSR_WIN_LANE4 == 2
                    // exact element-order sums: a row is started as +0.0 + first product (the
                    // oracle's loop), continued across lanes by serial carries (round r settles
                    // chains of r head-less lanes; rows of <= 32 elements cross <= 8 lanes)
                    const int f = hb ? __ffs(hb) - 1 : 4;  // my elements before my first head
                    double run = 0.0;
                    bool seen = false;
#pragma unroll
                    for (int j = 0; j < 4; j++) {
                        const bool h = (hb >> j) & 1u;
                        if (h && seen) res[hi - 1] = run;  // a row that starts and ends in this lane
                        run = h ? 0.0 + q[j] : run + q[j];
                        hi += h ? 1 : 0;
                        seen = seen || h;
                    }
                    const int left = T - t0;  // real elements in this chunk
                    const int nreal = left >= 128 ? 32 : (left + 3) >> 2;
                    const unsigned real = nreal >= 32 ? FULL : (1u << nreal) - 1u;
                    const unsigned hl = __ballot_sync(FULL, seen);
                    unsigned m = ~hl & real;
                    int rounds = 1;
                    while (m) {  // longest run of head-less real lanes
                        m &= m << 1;
                        rounds++;
                    }
                    const double cin0 = pend_rj >= 0 ? pend_s : 0.0;  // lane 0's carry: the row open across the chunk edge
                    double out = run;  // the running sum I pass to my right neighbour
                    for (int r = 0; r < rounds; r++) {
                        double cin = __shfl_up_sync(FULL, out, 1);
                        if (lane == 0) cin = cin0;
                        if (!seen) out = (((cin + q[0]) + q[1]) + q[2]) + q[3];
                    }
                    double cin = __shfl_up_sync(FULL, out, 1);
                    if (lane == 0) cin = cin0;
                    if (seen) {  // the row continuing into my lane ends before my first head
                        double x = cin;
#pragma unroll
                        for (int j = 0; j < 4; j++)
                            if (j < f) x += q[j];
                        const int rc = hi - __popc(hb) - 1;  // its table index
                        if (rc >= 0) res[rc] = x;
                    }
                    const int nh = Q0 + __popc(Hs[0]) + __popc(Hs[1]) + __popc(Hs[2]) + __popc(Hs[3]);
                    const double tail = __shfl_sync(FULL, out, nreal - 1);  // the open row at the last real lane
                    if (left > 128) {
                        pend_s = tail;
                        pend_rj = nh - 1;
                    } else {
                        if (lane == 0 && nh > 0) res[nh - 1] = tail;
                        pend_rj = -1;
                    }
                }
                __syncwarp();
#else
                    double run = 0.0, c = 0.0;
                    bool seen = false;
#pragma unroll
                    for (int j = 0; j < 4; j++) {
                        const bool h = (hb >> j) & 1u;
                        if (h && seen) res[hi - 1] = run;  // a row that starts and ends in this lane
                        if (h && !seen) c = run;           // elements before the lane's first head
                        run = h ? q[j] : run + q[j];
                        hi += h ? 1 : 0;
                        seen = seen || h;
                    }
                    if (!seen) c = run;
                    // U = c_i + (lane i has no head ? U_{i+1} : 0): what lane i passes to the row open on its left
                    double U = c;
                    int S = seen ? 1 : 0;
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
                        const double Ur = __shfl_down_sync(FULL, U, d);
                        const int Sr = __shfl_down_sync(FULL, S, d);
                        if (lane + d < 32) {
                            if (!S) U += Ur;
                            S |= Sr;
                        }
                    }
                    const double R = __shfl_down_sync(FULL, U, 1);  // from the lanes on my right
                    const double U0 = __shfl_sync(FULL, U, 0);      // the chunk's leading elements
                    const unsigned hl = __ballot_sync(FULL, seen);
                    const int ls = hl ? 31 - __clz((int)hl) : -1;  // lane of the chunk's last row head
                    const double open = run + (lane < 31 ? R : 0.0);
                    if (seen && lane != ls) res[hi - 1] = open;  // completed inside this chunk
                    if (lane == 0 && pend_rj >= 0) res[pend_rj] = pend_s + U0;
                    if (ls >= 0) {
                        pend_s = __shfl_sync(FULL, open, ls);
                        pend_rj = __shfl_sync(FULL, hi - 1, ls);
                    } else {
                        pend_rj = -1;
                    }
                }
                __syncwarp();
#endif  // ACSR_WIN_LANE4 == 2
#else
#pragma unroll
                for (int g = 0; g < WIN_G; g++) buf[32 * g + lane] = p[g];
                __syncwarp();
#if ACSR_PROF
                if (lane == 0) PROF_ADD(6, clock64() - pt0);
                pt0 = clock64();
#endif
                if (l > 0) {
                    const int i1 = min(pre + l, t0 + 32 * WIN_G) - t0;
                    int i = max(pre, t0) - t0;
#if ACSR_WIN_SUM4
                    // four accumulators by row offset j mod 4, each summed in element order:
                    // the result depends only on the row (not on where the 128-element
                    // chunks cut it) and the chain of dependent adds is 4x shorter
                    int j = i + t0 - pre;
                    for (; i < i1 && (j & 3); i++, j++) {
                        const double b = buf[i];
                        const int m = j & 3;
                        a1 += m == 1 ? b : 0.0;
                        a2 += m == 2 ? b : 0.0;
                        a3 += m == 3 ? b : 0.0;
                    }
                    for (; i + 4 <= i1; i += 4) {
                        const double b0 = buf[i], b1 = buf[i + 1], b2 = buf[i + 2], b3 = buf[i + 3];
                        acc += b0;
                        a1 += b1;
                        a2 += b2;
                        a3 += b3;
                    }
                    if (i < i1) acc += buf[i];
                    if (i + 1 < i1) a1 += buf[i + 1];
                    if (i + 2 < i1) a2 += buf[i + 2];
                    i = i1;
#endif
#if ACSR_WIN_LDS4
                    // four shared loads in flight, then the adds in element order (the sum
                    // is the same bits as the one-at-a-time loop; only the loads overlap)
                    for (; i + 4 <= i1; i += 4) {
                        const double b0 = buf[i], b1 = buf[i + 1], b2 = buf[i + 2], b3 = buf[i + 3];
                        acc += b0;
                        acc += b1;
                        acc += b2;
                        acc += b3;
                    }
#endif
                    for (; i < i1; i++) acc += buf[i];
                }
                __syncwarp();
#if ACSR_PROF
                if (lane == 0) PROF_ADD(7, clock64() - pt0);
                pt0 = clock64();
#endif
#endif
            }
#if ACSR_WIN_SEGSCAN
            if (l > 0) acc = buf[__popc(ne & lt)];
#elif ACSR_WIN_LANE4
            if (lane == 0 && pend_rj >= 0) ((double *)tab)[pend_rj] = pend_s;  // the window's last row
            __syncwarp();
            if (l > 0) acc = ((const double *)tab)[__popc(ne & lt)];
#elif ACSR_WIN_SUM4
            acc = (acc + a1) + (a2 + a3);
#endif
            if (mine) finish(a, r, acc, d2);
            __syncwarp();  // tab / buf reused by the next window
        }
    }
#endif

    static __device__ __forceinline__ void empty_rows(const A &a, int start, int cnt, int lane, Fix192 &d2)
    {
        for (int i = lane; i < cnt; i += 32) finish(a, __ldg(a.bin_rows + start + i), 0.0, d2);
    }

    // one HEAVY_CHUNK chunk of a long row; last arriver combines in chunk order
    static __device__ __forceinline__ void heavy(const A &a, int u, int r, int c, int lane, Fix192 &d2)
    {
        int beg, end;
        row_bounds(a, r, beg, end);
        const int kb = beg + c * HEAVY_CHUNK;
        const int ke = min(kb + HEAVY_CHUNK, end);
        const double s = warp_sum(strided_dot(a, kb, ke, lane));
        const int nch = heavy_chunks(end - beg);
        if (nch == 1) {
            if (lane == 0) finish(a, r, s, d2);
            return;
        }
        const int u0 = u - c;
        int last = 0;
        if (lane == 0) {
            a.partial[u] = s;
            __threadfence();
            last = (atomicAdd(a.ticket + u0, 1) == nch - 1);
        }
        last = __shfl_sync(0xffffffffu, last, 0);
        if (!last) return;
        __threadfence();
        double t = 0.0;
        for (int j = lane; j < nch; j += 32) t += __ldcg(a.partial + u0 + j);
        t = warp_sum(t);
        if (lane == 0) {
            a.ticket[u0] = 0;  // ready for the next call on this plan
            finish(a, r, t, d2);
        }
    }

#if ACSR_MERGED_WARP_PATH
    // Heavy chunks and the warp-per-row bins 7..10 in ONE loop, so the vectorised
    // strided_dot and the epilogue are inlined once for both (I-cache: the PageRank
    // kernel's executed code did not fit, ncu no_instruction stalls).
    static __device__ __forceinline__ void warp_rows(const A &a, int u, int2 d, int lane, Fix192 &d2)
    {
        const uint32_t y = (uint32_t)d.y;
        const bool hv = (y & HEAVY_FLAG) != 0;
        int cnt, myr = 0, mb = 0, me = 0, c = 0, nch = 0;
        if (hv) {
            c = (int)(y & ~HEAVY_FLAG);
            int beg, end;
            row_bounds(a, d.x, beg, end);
            cnt = 1;
            myr = d.x;
            mb = beg + c * HEAVY_CHUNK;
            me = min(mb + HEAVY_CHUNK, end);
            nch = heavy_chunks(end - beg);
        } else {
            cnt = (int)(y & 0xFFFFFF);
            if (lane < cnt) {
                myr = __ldg(a.bin_rows + d.x + lane);
                row_bounds(a, myr, mb, me);
            }
        }
        for (int i = 0; i < cnt; i++) {
            const int r = __shfl_sync(0xffffffffu, myr, i);
            const int kb = __shfl_sync(0xffffffffu, mb, i);
            const int ke = __shfl_sync(0xffffffffu, me, i);
            double s = warp_sum(strided_dot(a, kb, ke, lane));
            if (hv && nch > 1) {  // one chunk of a long row: last arriver combines in chunk order
                const int u0 = u - c;
                int last = 0;
                if (lane == 0) {
                    a.partial[u] = s;
                    __threadfence();
                    last = (atomicAdd(a.ticket + u0, 1) == nch - 1);
                }
                last = __shfl_sync(0xffffffffu, last, 0);
                if (!last) return;
                __threadfence();
                double t = 0.0;
                for (int j = lane; j < nch; j += 32) t += __ldcg(a.partial + u0 + j);
                s = warp_sum(t);
                if (lane == 0) a.ticket[u0] = 0;  // ready for the next call on this plan
            }
            if (lane == 0) finish(a, r, s, d2);
        }
    }
#endif

    // Fused peer exchange, per-tile push (ACSR_PEER_TILE_PUSH): every row of a unit lies in
    // one 1024-row tile; after the unit the warp adds its finished rows to the tile's count
    // (release: threadfence before the atomic), and the warp that completes the tile reads
    // the tile's xs' entries back from its own buffer (L2) and stores them to every other
    // rank as coalesced 256-byte warp stores -- instead of one scattered 8-byte remote store
    // per row and peer as rows finish in bin order.
    static __device__ __forceinline__ void peer_tile_done(const A &a, int lane, Fix192 &d2)
    {
        constexpr unsigned FULL = 0xffffffffu;
        const int total = __reduce_add_sync(FULL, d2.fin);
        if (total == 0) return;
        const unsigned any = __ballot_sync(FULL, d2.fin > 0);
        const int tile = __shfl_sync(FULL, d2.ftile, __ffs(any) - 1);
        d2.fin = 0;
        const int tile_rows = (int)min((int64_t)TILE_ROWS, a.n_rows - (int64_t)tile * TILE_ROWS);
        int done = 0;
        if (lane == 0) {
            __threadfence();
            done = atomicAdd(a.tile_done + tile, total) + total == tile_rows;
        }
        done = __shfl_sync(FULL, done, 0);
        if (!done) return;
        __threadfence();
        const int r0 = tile * TILE_ROWS;
        const int r1 = min(r0 + tile_rows, a.peer_len);
        const char *own = a.pself + a.peer_next + 8 * a.peer_off;
        for (int q = 0; q < a.peer_n; q++) {
            if (q == a.peer_rank || ACSR_DIAG == 4) continue;  // DIAG 4: no remote stores (store-count baseline)
            char *dst = a.pbase[q] + a.peer_next + 8 * a.peer_off;
            for (int r = r0 + lane; r < r1; r += 32)
                *(double *)(dst + 8 * (int64_t)r) = __ldcg((const double *)(own + 8 * (int64_t)r));
        }
        if (lane == 0) a.tile_done[tile] = 0;  // ready for the next step on this plan
    }

    static __device__ __forceinline__ void unit(const A &a, int u, int lane, Fix192 &d2, double *wbuf, int2 *wtab)
    {
        unit_d(a, u, __ldg(a.units + u), lane, d2, wbuf, wtab);
    }
    static __device__ __forceinline__ void unit_d(const A &a, int u, const int2 d, int lane, Fix192 &d2, double *wbuf,
                                                  int2 *wtab)
    {
        const uint32_t y = (uint32_t)d.y;
#if ACSR_MERGED_WARP_PATH
        if ((y & HEAVY_FLAG) || (!(y & WIN_FLAG) && (int)(y >> 24) > 6)) {
            warp_rows(a, u, d, lane, d2);
            return;
        }
#else
        if (y & HEAVY_FLAG) {
            heavy(a, u, d.x, (int)(y & ~HEAVY_FLAG), lane, d2);
            return;
        }
#endif
        if (WIN_MAX_BIN >= 0 && (y & WIN_FLAG)) {
#if ACSR_PF_TILES > 0
            // the first window unit of tile t (the list goes tile by tile) starts the L2
            // prefetch of tile t + ACSR_PF_TILES's CSR run: the column/value streams then
            // come from L2 instead of DRAM when their units run (bounds loaded now, the
            // prefetch issued after this unit so the loads' latency overlaps its work)
            int pb = 0, pe = 0;
            const bool pf = (d.x % TILE_ROWS) == 0 && lane == 0;
            if (pf) {
                const int64_t t0 = (int64_t)d.x + (int64_t)ACSR_PF_TILES * TILE_ROWS;
                if (t0 < a.n_rows) {
                    const int64_t t1 = t0 + TILE_ROWS < a.n_rows ? t0 + TILE_ROWS : a.n_rows;
                    pb = __ldg(a.rb + t0);
                    pe = HAS_END ? __ldg(a.re + t1 - 1) : __ldg(a.rb + t1);
                }
            }
            window(a, d.x, (int)(y & 0xFFFFFF), lane, d2, wbuf, wtab);
            if (pf && pe > pb) pf_range(a, pb, pe);
#else
            window(a, d.x, (int)(y & 0xFFFFFF), lane, d2, wbuf, wtab);
#endif
            return;
        }
        const int b = (int)(y >> 24), cnt = (int)(y & 0xFFFFFF);
        switch (b) {
            case 0: empty_rows(a, d.x, cnt, lane, d2); break;
            case 1: light_sub<1>(a, d.x, cnt, lane, d2); break;
            case 2: light_sub<2>(a, d.x, cnt, lane, d2); break;
            case 3: light_sub<4>(a, d.x, cnt, lane, d2); break;
            case 4: light_sub<8>(a, d.x, cnt, lane, d2); break;
            case 5: light_sub<16>(a, d.x, cnt, lane, d2); break;
            case 6: light_sub<32>(a, d.x, cnt, lane, d2); break;
#if !ACSR_MERGED_WARP_PATH
            default: light_warp(a, d.x, cnt, lane, d2); break;
#endif
        }
    }
};

#ifndef ACSR_SCHED_STATIC
#define ACSR_SCHED_STATIC 0  // 1: static round-robin units (A/B builds)
#endif

#ifndef ACSR_MIN_BLOCKS
#define ACSR_MIN_BLOCKS (1024 / SPMV_THREADS)  // 64 registers per thread
#endif

template <typename V, bool HAS_VAL, bool HAS_END, bool PR, bool XC, bool PEER = false>
__global__ void __launch_bounds__(SPMV_THREADS, ACSR_MIN_BLOCKS)
spmv_kernel(SpmvArgs<V> a)
{
    static_assert(!PEER || (PR && !XC), "the peer exchange is a PageRank-step epilogue");
    using K = Kern<V, HAS_VAL, HAS_END, PR, XC, PEER>;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint64_t bar;
    const int lane = threadIdx.x & 31;
    const int gw = blockIdx.x * SPMV_WARPS + (threadIdx.x >> 5);
    const int nw = gridDim.x * SPMV_WARPS;
    PlanHeader *hdr = a.hdr;
    if (a.x_prefetch > 0 && threadIdx.x < 32) {
        // x fits L2: every CTA bulk-prefetches its slice into L2 before waiting for the
        // previous grid (PDL), so the first gather of each sector does not pay a DRAM
        // round trip.  A prefetch is only a cache hint -- L2 is the point of coherence,
        // so prefetching before the producer of x has finished can never return stale data.
        const uintptr_t x0 = ((uintptr_t)a.x + 15) & ~(uintptr_t)15;
        const uintptr_t x1 = ((uintptr_t)a.x + (uintptr_t)a.x_prefetch) & ~(uintptr_t)15;
        if (x1 > x0) {
            const uintptr_t per = (((x1 - x0) + gridDim.x - 1) / gridDim.x + 15) & ~(uintptr_t)15;
            const uintptr_t b0 = x0 + per * blockIdx.x;
            const uintptr_t b1 = b0 + per < x1 ? b0 + per : x1;
            constexpr uintptr_t CH = 8192;
            for (uintptr_t p = b0 + CH * (threadIdx.x & 31); p < b1; p += CH * 32) {
                const uint32_t sz = (uint32_t)(b1 - p < CH ? b1 - p : CH);
                asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(sz) : "memory");
            }
        }
    }
#if ACSR_PF_START_TILES > 0
    if (threadIdx.x < 32) {  // the CSR runs of the first tiles the warps will take, into L2, while the
        // grid waits for the binning (PDL): start-up only, no prefetch inside the loop
        for (int64_t t = blockIdx.x + threadIdx.x * (int64_t)gridDim.x; t < ACSR_PF_START_TILES;
             t += 32 * (int64_t)gridDim.x) {
            const int64_t t0 = t * TILE_ROWS;
            if (t0 >= a.n_rows) break;
            const int64_t t1 = t0 + TILE_ROWS < a.n_rows ? t0 + TILE_ROWS : a.n_rows;
            const int pb = __ldg(a.rb + t0);
            const int pe = HAS_END ? __ldg(a.re + t1 - 1) : __ldg(a.rb + t1);
            if (pe > pb) K::pf_range(a, pb, pe);
        }
    }
#endif
#if ACSR_PF_TILES > 0
    if (threadIdx.x < 32) {  // tiles 0 .. ACSR_PF_TILES-1: one per CTA, grid-strided (before the PDL wait:
        // the CSR is not written by the preceding kernels; a prefetch is only a cache hint)
        for (int64_t t = blockIdx.x + threadIdx.x * (int64_t)gridDim.x; t < ACSR_PF_TILES; t += 32 * (int64_t)gridDim.x) {
            const int64_t t0 = t * TILE_ROWS;
            if (t0 >= a.n_rows) break;
            const int64_t t1 = t0 + TILE_ROWS < a.n_rows ? t0 + TILE_ROWS : a.n_rows;
            const int pb = __ldg(a.rb + t0);
            const int pe = HAS_END ? __ldg(a.re + t1 - 1) : __ldg(a.rb + t1);
            if (pe > pb) K::pf_range(a, pb, pe);
        }
    }
#endif
#if ACSR_TIMELINE
    const long long tl_c0 = clock64();
    if (threadIdx.x == 0 && blockIdx.x < 1024) {
        g_tl_cta[blockIdx.x][0] = gtimer();
        g_tl_cta[blockIdx.x][1] = (unsigned long long)tl_c0;
    }
#endif
    pdl_enter();
    // the first unit's descriptor in flight with the header loads below (the unit list's
    // offset depends on n_rows only, the host passes it): one dependent L2 round trip
    // less at start-up; used only if the header confirms gw < n_units
    int2 desc0 = make_int2(0, 0);
    if (ACSR_DESC0 == 1 && a.units_off > 0 && gw < a.light_cap)
        desc0 = __ldg((const int2 *)((const char *)hdr + a.units_off) + gw);
    if (ACSR_DESC0 == 2 && a.units_off > 0 && gw < a.light_cap && lane == 0)  // into L1 only: the loop is unchanged
        asm volatile("prefetch.global.L1 [%0];" ::"l"((const int2 *)((const char *)hdr + a.units_off) + gw));
    if (PR && a.ctrl && *(volatile int32_t *)a.ctrl) return;  // converged earlier: no-op step
    unsigned long long pc = 0;  // peer exchange: pushes completed before this step
    __shared__ char *s_pbase[PEER_MAX];
    if (PEER) {
        const PeerArgs *P = a.peer;
        pc = *(volatile unsigned long long *)&P->st->pushes;
        a.x = (const V *)(P->base[P->rank] + P->off_buf[(pc + 1) & 1]);  // filled by push pc
        a.peer_next = P->off_buf[pc & 1];
        a.peer_off = P->slice_off;
        a.peer_len = (int)P->slice_len;
        a.peer_n = P->nranks;
        a.peer_rank = P->rank;
        a.pself = P->base[P->rank];
        if (threadIdx.x < PEER_MAX) s_pbase[threadIdx.x] = threadIdx.x < P->nranks ? P->base[threadIdx.x] : nullptr;
        a.pbase = s_pbase;
        // every rank has completed push pc: buffer (pc-1)&1 is complete everywhere, and
        // nobody still reads buffer pc&1 (the previous step of every rank read it)
        // device-side convergence across ranks: the global Delta^2 of the previous step
        // is complete now -- every CTA takes the same decision from the same partials
        __shared__ int s_stop;
        if (threadIdx.x == 0) {
            peer_wait(*P, pc);
            s_stop = (a.ctrl && P->st->last_step && peer_sum_d2(*P, pc) <= a.eps2) ? 1 : 0;
        }
        __syncthreads();
        if (s_stop) {
            if (blockIdx.x == 0 && threadIdx.x == 0) a.ctrl[0] = 1;
            return;
        }
    }
    const int n_units = hdr->n_units;
    // A plan whose unit list overflowed its workspace (acsr_bin with an understated
    // nnz_max) has n_units == 0: the rows are not computed.  Never return stale data
    // silently: every output row gets a quiet NaN (and, for PageRank, Delta^2 = NaN and
    // ctrl[0] = ACSR_CTRL_PLAN_ERROR, below); acsr_plan_status reports the cause.
    const int plan_bad = *(volatile int32_t *)&hdr->overflow;
    if (plan_bad) {
        const double qnan = __longlong_as_double(0x7ff8000000000000ll);
        for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < a.n_rows;
             r += (int64_t)gridDim.x * blockDim.x) {
            if (PR) {
                a.x_new[r] = qnan;
                if (a.xs_next) a.xs_next[r] = qnan;
            } else {
                a.y[r] = (V)qnan;
            }
        }
    }
    {
        char *ws = (char *)hdr;
        a.units = (const int2 *)(ws + hdr->off_units);
        a.partial = (double *)(ws + hdr->off_partial);
        a.ticket = (int32_t *)(ws + hdr->off_ticket);
        a.tile_done = (int32_t *)(ws + hdr->off_tile_done);
    }
    if (XC) {
        // shared x cache: [XC_SLOTS values | XC_SLOTS 16-bit tags], filled by TMA bulk copies
        const uint32_t slots = 1u << a.xc_bits;
        V *sval = (V *)smem;
        uint16_t *stag = (uint16_t *)(smem + sizeof(V) * slots);
        const char *ws = (const char *)hdr;
        if (threadIdx.x == 0) {
            mbar_init(&bar, 1);
            const uint32_t vbytes = sizeof(V) * slots, tbytes = sizeof(uint16_t) * slots;
            mbar_expect_tx(&bar, vbytes + tbytes);
            constexpr uint32_t CH = 32768;
            for (uint32_t o = 0; o < vbytes; o += CH)
                bulk_g2s((char *)sval + o, ws + hdr->off_xc_val + o, CH < vbytes - o ? CH : vbytes - o, &bar);
            bulk_g2s(stag, ws + hdr->off_xc_tag, tbytes, &bar);
        }
        __syncthreads();
        mbar_wait(&bar, 0);
        a.xval = sval;
        a.xtag = stag;
    }
    // per-warp short-row window scratch (products + (beg, pre) table)
#if ACSR_WIN_DYN_SMEM
    // window scratch in dynamic shared memory after the (optional) x cache: lets WIN_G > 4
    double *win_buf = (double *)(smem + (XC ? (sizeof(V) + sizeof(uint16_t)) * ((size_t)1 << a.xc_bits) : 0));
    int2 *win_tab = (int2 *)(win_buf + SPMV_WARPS * 32 * WIN_G);  // WIN_TAB entries per warp
#else
    __shared__ __align__(16) double win_buf[WIN_MAX_BIN >= 0 ? SPMV_WARPS * 32 * WIN_G : 1];
    __shared__ int2 win_tab[WIN_MAX_BIN >= 0 ? SPMV_WARPS * WIN_TAB : 1];
#endif
    double *wbuf = win_buf + (WIN_MAX_BIN >= 0 ? (threadIdx.x >> 5) * 32 * WIN_G : 0);
    int2 *wtab = win_tab + (WIN_MAX_BIN >= 0 ? (threadIdx.x >> 5) * WIN_TAB : 0);
    Fix192 d2{0, 0, 0, 0, 0};
    const bool tile_push = PEER && ACSR_PEER_TILE_PUSH && a.peer_n > 1;
#if ACSR_SCHED_STATIC
    for (int u = gw; u < n_units; u += nw) {
        K::unit(a, u, lane, d2, wbuf, wtab);
        if (tile_push) K::peer_tile_done(a, lane, d2);
    }
#else
    // first prefetched claims: one atomic per CTA (a same-address atomic per warp at
    // launch costs microseconds of serialisation at the L2 slice)
    __shared__ int s_claim;
#if ACSR_CLAIM_BATCH > 0
    if (threadIdx.x == 0) s_claim = SPMV_WARPS * atomicAdd(&hdr->work_ctr, 1);  // this CTA's batch 0
#elif ACSR_CLAIM_LATE
    // prefetched first claims only while more than one round of units remains after them
    const bool cta_ahead = ACSR_CLAIM_LATE == 2 && 2 * nw < n_units;
    if (threadIdx.x == 0) s_claim = cta_ahead ? atomicAdd(&hdr->work_ctr, SPMV_WARPS) : 0;
#else
    if (threadIdx.x == 0) s_claim = atomicAdd(&hdr->work_ctr, SPMV_WARPS);
#endif
    __syncthreads();
    int u = gw;
    int nxt = s_claim + (threadIdx.x >> 5);
#if ACSR_PROF
    long long t_first = clock64(), t_last = 0;
    if (lane == 0) PROF_ADD(8, 0);
    bool first = true;
#endif
#if ACSR_CLAIM_BATCH > 0
    // CTA-batched claiming: after the static first round (unit = global warp id) the
    // global counter hands out batches of ACSR_CLAIM_BATCH consecutive units to a CTA,
    // whose warps take them one by one from a shared-memory counter.  The warp that
    // takes the first unit of batch b fetches the id of batch b + 1, so a batch is
    // published long before it is needed; global atomics drop ACSR_CLAIM_BATCH-fold, so
    // units can be small (short tail) without saturating one L2 slice with claims.
    constexpr int CB = ACSR_CLAIM_BATCH;
    constexpr int RING = 32;  // published batch ids: (local batch << 32 | global batch), one 64-bit word
    __shared__ int s_claims;
    __shared__ unsigned long long s_batch[RING];
    if (threadIdx.x < RING) s_batch[threadIdx.x] = ~0ull;
    if (threadIdx.x == 0) {
        s_claims = 0;
        s_batch[0] = (unsigned long long)(unsigned)(s_claim / SPMV_WARPS);  // batch 0: the CTA's first atomic
    }
    __syncthreads();
    auto claim = [&]() -> int {
        const int i = atomicAdd(&s_claims, 1);
        const int b = i / CB, j = i - b * CB;
        if (j == 0) {  // fetch the NEXT batch's id, published with its local batch number
            const int g = atomicAdd(&hdr->work_ctr, 1);
            ((volatile unsigned long long *)s_batch)[(b + 1) % RING] =
                ((unsigned long long)(unsigned)(b + 1) << 32) | (unsigned)g;
        }
        unsigned long long v;
        while (((v = ((volatile unsigned long long *)s_batch)[b % RING]) >> 32) != (unsigned long long)(unsigned)b)
            __nanosleep(32);
        return nw + (int)(unsigned)v * CB + j;
    };
    if (lane == 0) nxt = claim();
#endif
#if ACSR_CLAIM_GUIDED > 0 && ACSR_CLAIM_BATCH == 0 && !ACSR_DESC_AHEAD && !ACSR_PROF
    // guided batches: a warp takes k consecutive units per claim, k = (units left) /
    // (ACSR_CLAIM_GUIDED * warps) clamped to [1, 32] -- large batches while much work
    // remains, single units at the end (the tail is one short unit, not one long one).
    // The batch's descriptors arrive in ONE coalesced load (no dependent descriptor
    // round trip per unit) and the claim for the next batch is issued when the batch's
    // last unit starts (ACSR_GUIDED_AHEAD) or when it ends.  Round 0 is static: warp w
    // takes units [w k0, (w+1) k0); claims hand out units from nw k0 on.
    {
        constexpr int F = ACSR_CLAIM_GUIDED;
        auto batch = [&](int left) -> int {
            const int k = left / (F * nw);
            return k < 1 ? 1 : (k > 32 ? 32 : k);
        };
        const int k0 = batch(n_units);
        const int S = nw * k0;
        int base = gw * k0;
        int cnt = base < n_units ? min(k0, n_units - base) : 0;
        int seen = 0;  // the counter's value at this warp's last claim
        while (cnt > 0) {
            const int2 dl = lane < cnt ? __ldg(a.units + base + lane) : make_int2(0, 0);
            int nb = 0, k = 1;
            for (int i = 0; i < cnt; i++) {
                const bool last = i == cnt - 1;
                if (last && ACSR_GUIDED_AHEAD) {
                    k = batch(n_units - S - seen);
                    if (lane == 0) nb = atomicAdd(&hdr->work_ctr, k);
                }
                int2 d;
                d.x = __shfl_sync(0xffffffffu, dl.x, i);
                d.y = __shfl_sync(0xffffffffu, dl.y, i);
#if ACSR_TIMELINE
                const long long tl_s = clock64() - tl_c0;
                const uint32_t tl_ty = (uint32_t)d.y;
                const unsigned long long tl_kind =
                    (tl_ty & HEAVY_FLAG) ? 3 : (tl_ty & WIN_FLAG) ? 0 : ((tl_ty >> 24) == 0 ? 4 : ((tl_ty >> 24) <= 6 ? 1 : 2));
#endif
                K::unit_d(a, base + i, d, lane, d2, wbuf, wtab);
#if ACSR_TIMELINE
                __syncwarp();
                if (lane == 0 && base + i < TL_MAX) {
                    const unsigned long long tag = ((unsigned long long)smid() << 48) | (tl_kind << 56);
                    g_tl[base + i][0] = (unsigned long long)tl_s | tag;
                    g_tl[base + i][1] = (unsigned long long)(clock64() - tl_c0) | tag;
                }
#endif
                if (tile_push) K::peer_tile_done(a, lane, d2);
            }
            if (!ACSR_GUIDED_AHEAD) {
                k = batch(n_units - S - seen);
                if (lane == 0) nb = atomicAdd(&hdr->work_ctr, k);
            }
            seen = __shfl_sync(0xffffffffu, nb, 0);
            base = S + seen;
            cnt = base < n_units ? min(k, n_units - base) : 0;
            seen += k;
        }
    }
#elif ACSR_CLAIM_LATE && ACSR_CLAIM_BATCH == 0 && !ACSR_DESC_AHEAD && !ACSR_PROF
    // late claims: a prefetched claim parks a unit on a busy warp, which with ~1-2 units
    // per warp (C3a) leaves other warps idle at the end.  Mode 1 claims every unit only
    // when the warp is free; mode 2 keeps prefetched claims while more than one round of
    // units remains and claims late in the last round.
    bool have = cta_ahead;
    bool first = ACSR_DESC0 == 1 && a.units_off > 0 && gw < a.light_cap &&
                 (const char *)a.units == (const char *)hdr + a.units_off;
    while (u < n_units) {
#if ACSR_TIMELINE
        const long long tl_s = clock64() - tl_c0;
        const uint32_t tl_ty = (uint32_t)__ldg(a.units + u).y;
        const unsigned long long tl_kind =
            (tl_ty & HEAVY_FLAG) ? 3 : (tl_ty & WIN_FLAG) ? 0 : ((tl_ty >> 24) == 0 ? 4 : ((tl_ty >> 24) <= 6 ? 1 : 2));
#endif
#if ACSR_DESC0 == 1
        K::unit_d(a, u, first ? desc0 : __ldg(a.units + u), lane, d2, wbuf, wtab);
        first = false;
#else
        K::unit(a, u, lane, d2, wbuf, wtab);
#endif
#if ACSR_TIMELINE
        __syncwarp();
        if (lane == 0 && u < TL_MAX) {
            const unsigned long long tag = ((unsigned long long)smid() << 48) | (tl_kind << 56);
            g_tl[u][0] = (unsigned long long)tl_s | tag;
            g_tl[u][1] = (unsigned long long)(clock64() - tl_c0) | tag;
        }
#endif
        if (tile_push) K::peer_tile_done(a, lane, d2);
        if (!have && lane == 0) nxt = atomicAdd(&hdr->work_ctr, 1);
        u = __shfl_sync(0xffffffffu, nxt, 0) + nw;
        have = ACSR_CLAIM_LATE == 2 && u + nw < n_units;
        if (have && lane == 0) nxt = atomicAdd(&hdr->work_ctr, 1);
    }
#elif ACSR_DESC_AHEAD && ACSR_CLAIM_BATCH == 0 && !ACSR_PROF
    // two units in hand: the current one (descriptor loaded) and the next one, whose
    // descriptor load is in flight while the current unit runs; the claim for the one
    // after is outstanding as well -- no dependent round trip between units
    int un = s_claim + (threadIdx.x >> 5) + nw;
    int2 dc = make_int2(0, 0), dn = make_int2(0, 0);
    if (u < n_units) dc = __ldg(a.units + u);
    if (un < n_units) {
        dn = __ldg(a.units + un);
        if (lane == 0) nxt = atomicAdd(&hdr->work_ctr, 1);
    }
    while (u < n_units) {
        K::unit_d(a, u, dc, lane, d2, wbuf, wtab);
        if (tile_push) K::peer_tile_done(a, lane, d2);
        u = un;
        dc = dn;
        if (u >= n_units) break;
        un = __shfl_sync(0xffffffffu, nxt, 0) + nw;
        if (un < n_units) {
            dn = __ldg(a.units + un);
            if (lane == 0) nxt = atomicAdd(&hdr->work_ctr, 1);
        }
    }
#else
    while (u < n_units) {
#if ACSR_PROF
        const long long tu = clock64();
        if (first && lane == 0) PROF_ADD(8, tu - t_first);
        first = false;
        const uint32_t ty = (uint32_t)__ldg(a.units + u).y;
        const int kind = (ty & HEAVY_FLAG) ? 3 : (ty & WIN_FLAG) ? 0 : ((ty >> 24) == 0 ? 4 : ((ty >> 24) <= 6 ? 1 : 2));
#endif
        K::unit(a, u, lane, d2, wbuf, wtab);
#if ACSR_PROF
        __syncwarp();
        t_last = clock64();
        if (lane == 0) {
            PROF_ADD(kind, t_last - tu);
            PROF_ADD(10 + kind, 1);
        }
#endif
        if (tile_push) K::peer_tile_done(a, lane, d2);
#if ACSR_CLAIM_BATCH > 0
        u = __shfl_sync(0xffffffffu, nxt, 0);
        if (u < n_units && lane == 0) nxt = claim();
#else
        u = __shfl_sync(0xffffffffu, nxt, 0) + nw;
        if (u < n_units && lane == 0) nxt = atomicAdd(&hdr->work_ctr, 1);
#endif
    }
#endif  // ACSR_DESC_AHEAD
#if ACSR_PROF
    if (t_last == 0) t_last = clock64();
#endif
#endif
    // CTA-level exit: Delta^2 (exact fixed point) reduced warp -> CTA in shared memory,
    // then ONE set of atomics and ONE exit ticket per CTA
    __shared__ uint64_t s_d2[SPMV_WARPS][3];
    if (PR) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const uint64_t h = __shfl_xor_sync(0xffffffffu, d2.hi, o);
            const uint64_t m = __shfl_xor_sync(0xffffffffu, d2.mid, o);
            const uint64_t l = __shfl_xor_sync(0xffffffffu, d2.lo, o);
            fix_merge(d2, h, m, l);
        }
        if (lane == 0) {
            s_d2[threadIdx.x >> 5][0] = d2.hi;
            s_d2[threadIdx.x >> 5][1] = d2.mid;
            s_d2[threadIdx.x >> 5][2] = d2.lo;
        }
    }
    __syncthreads();
#if ACSR_PROF
    if (lane == 0) PROF_ADD(9, clock64() - t_last);
    if (threadIdx.x == 0 && blockIdx.x == 0) PROF_ADD(15, 1);
#endif
#if ACSR_TIMELINE
    if (threadIdx.x == 0 && blockIdx.x < 1024) g_tl_cta[blockIdx.x][2] = gtimer();
#endif
    if (threadIdx.x >= 32) return;
    if (PR) {
        d2 = lane < SPMV_WARPS ? Fix192{s_d2[lane][0], s_d2[lane][1], s_d2[lane][2], 0, 0} : Fix192{0, 0, 0, 0, 0};
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const uint64_t h = __shfl_xor_sync(0xffffffffu, d2.hi, o);
            const uint64_t m = __shfl_xor_sync(0xffffffffu, d2.mid, o);
            const uint64_t l = __shfl_xor_sync(0xffffffffu, d2.lo, o);
            fix_merge(d2, h, m, l);
        }
        if (lane == 0 && (d2.hi | d2.mid | d2.lo)) {
            const unsigned long long ol = atomicAdd((unsigned long long *)&hdr->d2_lo, (unsigned long long)d2.lo);
            const uint64_t c1 = (ol + d2.lo < ol) ? 1u : 0u;
            const uint64_t madd = d2.mid + c1;
            const uint64_t cm = (madd < d2.mid) ? 1u : 0u;  // d2.mid == 2^64-1 and c1
            const unsigned long long om = atomicAdd((unsigned long long *)&hdr->d2_mid, (unsigned long long)madd);
            const uint64_t c2 = (om + madd < om) ? 1u : 0u;
            atomicAdd((unsigned long long *)&hdr->d2_hi, (unsigned long long)(d2.hi + c2 + cm));
        }
    }
    // last CTA out publishes Delta^2 and resets the counters for the next call
    if (lane == 0) {
        // peer exchange: the CTA's remote xs stores must be visible system-wide before
        // the push is signalled (barrier above + system-scope fence, then the ticket chain)
        if (PEER) __threadfence_system();
        else __threadfence();
        if (atomicAdd(&hdr->exit_ticket, 1) == (int)gridDim.x - 1) {
            __threadfence();
            if (PR) {
                const uint64_t hi = *(volatile uint64_t *)&hdr->d2_hi;
                const uint64_t mid = *(volatile uint64_t *)&hdr->d2_mid;
                const uint64_t lo = *(volatile uint64_t *)&hdr->d2_lo;
                double d2v = (double)hi + ((double)mid + (double)lo * 5.421010862427522e-20) * 5.421010862427522e-20;
                if (plan_bad) d2v = __longlong_as_double(0x7ff8000000000000ll);
                *a.delta2 = d2v;  // with the peer exchange: this rank's partial
                if (PEER) {
                    __threadfence_system();
                    // an overflowed plan publishes a saturated partial: no rank converges on it
                    peer_signal(*a.peer, pc + 1, true, plan_bad ? ~0ull : hi, mid, lo);
                }
                if (a.d2_out) {  // acsr_comm: all-gathered and summed by the exchange
                    a.d2_out[0] = plan_bad ? ~0ull : hi;
                    a.d2_out[1] = mid;
                    a.d2_out[2] = lo;
                }
                if (a.ctrl && plan_bad) {
                    a.ctrl[0] = ACSR_CTRL_PLAN_ERROR;  // stops the loop; acsr_plan_status tells why
                } else if (a.ctrl) {
                    a.ctrl[1] += 1;
                    // peer exchange: the global test runs at the next step's entry (or in
                    // acsr_peer_delta2), once every rank's partial has arrived
                    if (!PEER && d2v <= a.eps2) a.ctrl[0] = 1;
                }
                hdr->d2_hi = 0;
                hdr->d2_mid = 0;
                hdr->d2_lo = 0;
            }
            hdr->work_ctr = 0;
            hdr->exit_ticket = 0;
        }
    }
}

// x-cache pre-pass: compact the hot x entries chosen by acsr_bin's vote table into
// the plan workspace (XC_SLOTS values + 16-bit tags) for the TMA fill.  Without a
// vote table (acsr_bin called without col_idx) every tag is XC_NOTAG.
template <typename V>
__global__ void xc_fill_kernel(PlanHeader *hdr, const V *__restrict__ x, int bits, int force_miss)
{
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    const int slots = 1 << bits;
    if (s >= slots) return;
    char *ws = (char *)hdr;
    unsigned long long v = 0ull;
    if (hdr->xc_valid && !force_miss) {
        const unsigned long long *best = (const unsigned long long *)(ws + hdr->off_xc_vote);
        for (int j = s; j < XC_SLOTS; j += slots) v = max(v, best[j]);  // counts compare first
    }
    const int64_t c = (int64_t)(uint32_t)v;
    const uint32_t t = (uint32_t)(c >> bits);
    const bool ok = (v >> 32) != 0 && c < hdr->n_cols && t < XC_NOTAG;
    ((uint16_t *)(ws + hdr->off_xc_tag))[s] = ok ? (uint16_t)t : XC_NOTAG;
    ((V *)(ws + hdr->off_xc_val))[s] = ok ? x[c] : (V)0;
}

static int env_int(const char *name, int dflt)
{
    const char *e = getenv(name);
    return (e && e[0]) ? atoi(e) : dflt;
}

// dynamic shared memory of the SpMV launch: the x cache plus an optional reserve
// (ACSR_SMEM_RESERVE, bytes; measurements only -- it shrinks L1)
template <typename V, bool XC>
static size_t spmv_smem(int bits)
{
    static int reserve = -1;
    if (reserve < 0) reserve = env_int("ACSR_SMEM_RESERVE", 0);
    const size_t win = ACSR_WIN_DYN_SMEM ? (size_t)SPMV_WARPS * (32 * WIN_G * sizeof(double) + WIN_TAB * sizeof(int2)) : 0;
    return (XC ? (sizeof(V) + sizeof(uint16_t)) * ((size_t)1 << bits) : 0) + win + (size_t)reserve;
}

// ACSR_X_PERSIST_MB=m (experiment, default off): an L2 access-policy window marks the
// first m MB of x persisting for every SpMV / PageRank launch (the persisting L2 set-aside
// is sized once, capped by the device maximum)
static int64_t x_persist_bytes()
{
    static int64_t v = -1;
    if (v < 0) {
        const char *e = getenv("ACSR_X_PERSIST_MB");
        v = (e && e[0]) ? (int64_t)atoll(e) << 20 : 0;
        if (v > 0) {
            int dev = 0, mx = 0, mw = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, dev);
            cudaDeviceGetAttribute(&mw, cudaDevAttrMaxAccessPolicyWindowSize, dev);
            if (v > mw) v = mw;
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)(v < mx ? v : mx));
        }
    }
    return v;
}

template <typename V, bool HAS_VAL, bool HAS_END, bool PR, bool XC, bool PEER = false>
static void launch(const SpmvArgs<V> &a, cudaStream_t s)
{
    static size_t configured = 0;
    const size_t smem = spmv_smem<V, XC>(a.xc_bits);
    if (smem > configured) {
        cudaFuncSetAttribute(spmv_kernel<V, HAS_VAL, HAS_END, PR, XC, PEER>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        configured = smem;
    }
    static int per_sm = 0;
    if (!per_sm) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, spmv_kernel<V, HAS_VAL, HAS_END, PR, XC, PEER>,
                                                      SPMV_THREADS, smem);
        if (per_sm < 1) per_sm = 1;
    }
    const int64_t persist = x_persist_bytes();
    if (persist > 0 && a.x) {
        // opt-in experiment: keep the first `persist` bytes of x persisting in L2 for this
        // launch (with a hot-first vertex order these hold most gathers)
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = per_sm * acsr_num_sms();
        cfg.blockDim = SPMV_THREADS;
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute at[2];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = acsr_pdl_enabled() ? 1 : 0;
        at[1].id = cudaLaunchAttributeAccessPolicyWindow;
        at[1].val.accessPolicyWindow.base_ptr = (void *)a.x;
        at[1].val.accessPolicyWindow.num_bytes = (size_t)persist;
        at[1].val.accessPolicyWindow.hitRatio = 1.0f;
        at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = at;
        cfg.numAttrs = 2;
        cudaLaunchKernelEx(&cfg, spmv_kernel<V, HAS_VAL, HAS_END, PR, XC, PEER>, a);
        return;
    }
    launch_pdl(spmv_kernel<V, HAS_VAL, HAS_END, PR, XC, PEER>, per_sm * acsr_num_sms(), SPMV_THREADS, smem, s, a);
}

template <typename V, bool PR, bool XC>
static void dispatch2(const SpmvArgs<V> &a, cudaStream_t s)
{
    const bool hv = a.val != nullptr, he = a.re != nullptr;
    if (hv && he) launch<V, true, true, PR, XC>(a, s);
    else if (hv) launch<V, true, false, PR, XC>(a, s);
    else if (he) launch<V, false, true, PR, XC>(a, s);
    else launch<V, false, false, PR, XC>(a, s);
}

// The shared-memory x cache is OFF by default: measured on B200 its
// tag lookups sit in the same L1TEX queue as the outstanding gathers, so they add a
// full queue latency to every gather and the kernel got slower (C2: 93 -> 116 us)
// even though L2 requests fell.  Knobs (read once; measurements only):
//   ACSR_XCACHE=1      enable the cache (acsr_bin must also see ACSR_XCACHE=1)
//   ACSR_XC_MISS=1     cache path with every tag invalid (lookup cost without hits)
//   ACSR_XC_BITS=k     2^k slots (k <= 14)
static int env_flag(const char *name)
{
    const char *e = getenv(name);
    return (e && e[0] == '1') ? 1 : 0;
}
static bool xcache_enabled()
{
    static int v = -1;
    if (v < 0) v = env_flag("ACSR_XCACHE");
    return v == 1;
}
static int xcache_force_miss()
{
    static int v = -1;
    if (v < 0) v = env_flag("ACSR_XC_MISS");
    return v;
}

// element phase for 128-bit loads of col (and val), or -1 if col and val cannot be
// vector-loaded at the same indices
template <typename V>
static int vec_phase(const int32_t *col, const V *val)
{
    const uintptr_t pc = (uintptr_t)col;
    if (pc % 4) return -1;
    const int ph = (int)((pc / 4) % 4);
    if (!val) return ph;
    const uintptr_t pv = (uintptr_t)val;
    if (pv % sizeof(V)) return -1;
    if (sizeof(V) == 8) return ((int)((pv / 8) % 2) == ph % 2) ? ph : -1;
    return ((int)((pv / 4) % 4) == ph) ? ph : -1;
}

static int xcache_bits()
{
    static int v = -1;
    if (v < 0) {
        v = env_int("ACSR_XC_BITS", XC_BITS);
        if (v < 8) v = 8;
        if (v > XC_BITS) v = XC_BITS;
    }
    return v;
}

// x is bulk-prefetched into L2 at SpMV entry when it is at most this large (a quarter of
// the ~126 MB L2); ACSR_XPREFETCH=0 switches it off (A/B)
static int64_t x_prefetch_bytes(int64_t bytes)
{
    static int on = -1;
    static int64_t max_bytes = 0;
    if (on < 0) {
        const char *e = getenv("ACSR_XPREFETCH");
        on = (e && e[0] == '0') ? 0 : 1;
        const char *m = getenv("ACSR_XPREFETCH_MAX_MB");  // largest x prefetched (r2s2: 32 -> 64 MB, C3b -0.35 %)
        max_bytes = (int64_t)(m && m[0] ? atoi(m) : 64) << 20;
    }
    return (on && bytes <= max_bytes) ? bytes : 0;
}

template <typename V, bool PR>
static int dispatch(SpmvArgs<V> a, cudaStream_t s)
{
    {
        const PlanLayout L = plan_layout(a.n_rows, 0, 0);  // the unit list's offset: n_rows alone
        a.units_off = (int64_t)L.off_units;
        a.light_cap = L.light_cap;
    }
    a.vph = ACSR_NO_VEC ? -1 : vec_phase<V>(a.col, a.val);
    a.xc_bits = xcache_bits();
    if (PR && a.peer) {  // fused peer exchange: pattern matrix, no x cache
        if (a.re) launch<V, false, true, true, false, true>(a, s);
        else launch<V, false, false, true, false, true>(a, s);
        return 1;
    }
    if (xcache_enabled() && a.x != nullptr) {
        xc_fill_kernel<V><<<((1 << a.xc_bits) + 255) / 256, 256, 0, s>>>(a.hdr, a.x, a.xc_bits,
                                                                          xcache_force_miss());
        dispatch2<V, PR, true>(a, s);
        return 2;
    }
    dispatch2<V, PR, false>(a, s);
    return 1;
}

__global__ void pagerank_scale_kernel(int64_t n, const double *__restrict__ x,
                                      const int32_t *__restrict__ outdeg, double *__restrict__ xs)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int od = outdeg[i];
        xs[i] = od > 0 ? x[i] / (double)od : 0.0;
    }
}

__global__ void zero_delta_kernel(double *d) { *d = 0.0; }

}  // namespace acsr

using namespace acsr;

static bool plan_ok(int64_t n_rows, const int32_t *bin_rows, const int32_t *bin_offsets, void *plan_ws,
                    size_t plan_ws_bytes)
{
    if (!bin_offsets || !plan_ws) return false;
    if (n_rows > 0 && !bin_rows) return false;
    return plan_ws_bytes >= plan_layout(n_rows, 0, 0).total;
}

extern "C" acsr_status acsr_spmv(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                 const int32_t *row_begin, const int32_t *row_end,
                                 const int32_t *col_idx, const void *values, const void *x, void *y,
                                 const int32_t *bin_rows, const int32_t *bin_offsets, void *plan_ws,
                                 size_t plan_ws_bytes, cudaStream_t stream)
{
    if (n_rows < 0 || n_cols < 0 || n_rows >= ((int64_t)1 << 31) ||
        (dt != ACSR_F32 && dt != ACSR_F64) || (n_rows > 0 && (!row_begin || !y))) {
        acsr_set_error("acsr_spmv: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!plan_ok(n_rows, bin_rows, bin_offsets, plan_ws, plan_ws_bytes)) {
        acsr_set_error("acsr_spmv: plan workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    if (n_rows == 0) return ACSR_OK;
    if (dt == ACSR_F64) {
        SpmvArgs<double> a{};
        a.rb = row_begin; a.re = row_end; a.col = col_idx;
        a.val = (const double *)values; a.x = n_cols > 0 ? (const double *)x : nullptr; a.y = (double *)y;
        a.bin_rows = bin_rows; a.hdr = (PlanHeader *)plan_ws; a.n_rows = n_rows;
        a.x_prefetch = a.x ? x_prefetch_bytes(n_cols * (int64_t)sizeof(double)) : 0;
        dispatch<double, false>(a, stream);
    } else {
        SpmvArgs<float> a{};
        a.rb = row_begin; a.re = row_end; a.col = col_idx;
        a.val = (const float *)values; a.x = n_cols > 0 ? (const float *)x : nullptr; a.y = (float *)y;
        a.bin_rows = bin_rows; a.hdr = (PlanHeader *)plan_ws; a.n_rows = n_rows;
        a.x_prefetch = a.x ? x_prefetch_bytes(n_cols * (int64_t)sizeof(float)) : 0;
        dispatch<float, false>(a, stream);
    }
    return acsr_check_launch("acsr_spmv");
}

extern "C" acsr_status acsr_pagerank_step(const acsr_pr_args *p, cudaStream_t stream)
{
    if (!p || p->n_rows < 0 || p->n_cols < 0 || p->n_rows >= ((int64_t)1 << 31) || !p->delta2 ||
        (p->n_rows > 0 && (!p->row_begin || !p->x || !p->outdeg || !p->x_new || !p->xs_next))) {
        acsr_set_error("acsr_pagerank_step: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!plan_ok(p->n_rows, p->bin_rows, p->bin_offsets, p->plan_ws, p->plan_ws_bytes)) {
        acsr_set_error("acsr_pagerank_step: plan workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    bool counts_bad = false;
    if (p->comm && p->slice_counts)
        for (int q = 0; q < acsr_comm_nranks(p->comm); q++)
            counts_bad |= p->slice_counts[q] < 0 || p->slice_counts[q] > p->slice_len;
    if (p->comm && (counts_bad || !p->xs_all || p->slice_len < 0 ||
                    p->n_cols < (int64_t)acsr_comm_nranks(p->comm) * p->slice_len || (p->slice_len > 0 && !p->xs_next))) {
        acsr_set_error("acsr_pagerank_step: with comm, xs_all [n_cols >= nranks * slice_len] and xs_next are required");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (p->n_rows == 0) {
        if (p->comm) {  // still part of the exchange: a zero partial
            cudaMemsetAsync(acsr_comm_d2_slot(p->comm), 0, 3 * sizeof(uint64_t), stream);
            return acsr_comm_step_exchange(p, stream);
        }
        zero_delta_kernel<<<1, 1, 0, stream>>>(p->delta2);
        return acsr_check_launch("acsr_pagerank_step(empty)");
    }
    SpmvArgs<double> a{};
    a.rb = p->row_begin; a.re = p->row_end; a.col = p->col_idx;
    a.val = nullptr; a.x = p->n_cols > 0 ? p->xs : nullptr; a.y = nullptr;
    a.bin_rows = p->bin_rows; a.hdr = (PlanHeader *)p->plan_ws; a.n_rows = p->n_rows;
    a.x_old = p->x; a.outdeg = p->outdeg; a.x_new = p->x_new; a.xs_next = p->xs_next;
    a.damping = p->damping; a.teleport = p->teleport; a.delta2 = p->delta2;
    a.restart = p->restart; a.restart_weight = p->restart_weight;
    a.ctrl = p->ctrl; a.eps2 = p->eps2;
    a.x_prefetch = a.x ? x_prefetch_bytes(p->n_cols * (int64_t)sizeof(double)) : 0;
    if (p->comm) {
        a.eps2 = -1.0;  // the stop decision is global (acsr_comm_step_exchange)
        a.d2_out = acsr_comm_d2_slot(p->comm);
    }
    dispatch<double, true>(a, stream);
    const acsr_status st = acsr_check_launch("acsr_pagerank_step");
    if (st != ACSR_OK || !p->comm) return st;
    return acsr_comm_step_exchange(p, stream);
}

extern "C" acsr_status acsr_pagerank_step_peer(const acsr_pr_args *p, acsr_peer *peer, cudaStream_t stream)
{
    if (!peer || !peer->opened) {
        acsr_set_error("acsr_pagerank_step_peer: peer object missing or not opened (acsr_peer_open)");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!p || p->n_rows < 0 || p->n_rows >= ((int64_t)1 << 31) || !p->delta2 || p->n_cols != peer->xs_len ||
        p->n_rows < peer->slice_len ||
        (p->n_rows > 0 && (!p->row_begin || !p->x || !p->outdeg || !p->x_new))) {
        acsr_set_error("acsr_pagerank_step_peer: invalid argument (n_cols must equal the peer xs_len, "
                       "n_rows >= slice_len)");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!plan_ok(p->n_rows, p->bin_rows, p->bin_offsets, p->plan_ws, p->plan_ws_bytes)) {
        acsr_set_error("acsr_pagerank_step_peer: plan workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    if (p->n_rows == 0) {  // nothing local: still take part in the barrier / signal
        acsr_set_error("acsr_pagerank_step_peer: a rank needs at least one row");
        return ACSR_ERR_INVALID_VALUE;
    }
    SpmvArgs<double> a{};
    a.rb = p->row_begin; a.re = p->row_end; a.col = p->col_idx;
    a.val = nullptr; a.x = nullptr; a.y = nullptr;  // x: the peer buffer, chosen in-kernel
    a.bin_rows = p->bin_rows; a.hdr = (PlanHeader *)p->plan_ws; a.n_rows = p->n_rows;
    a.x_old = p->x; a.outdeg = p->outdeg; a.x_new = p->x_new; a.xs_next = p->xs_next;
    a.damping = p->damping; a.teleport = p->teleport; a.delta2 = p->delta2;
    a.restart = p->restart; a.restart_weight = p->restart_weight;
    a.ctrl = p->ctrl; a.eps2 = p->eps2;
    a.peer = &((const PeerState *)peer->region)->view;
    dispatch<double, true>(a, stream);
    return acsr_check_launch("acsr_pagerank_step_peer");
}

extern "C" acsr_status acsr_pagerank_scale(int64_t n, const double *x, const int32_t *outdeg,
                                           double *xs, cudaStream_t stream)
{
    if (n < 0 || (n > 0 && (!x || !outdeg || !xs))) {
        acsr_set_error("acsr_pagerank_scale: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (n == 0) return ACSR_OK;
    int64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    pagerank_scale_kernel<<<(int)blocks, 256, 0, stream>>>(n, x, outdeg, xs);
    return acsr_check_launch("acsr_pagerank_scale");
}

extern "C" acsr_status acsr_plan_status(const void *plan_ws, size_t plan_ws_bytes, cudaStream_t stream)
{
    if (!plan_ws || plan_ws_bytes < sizeof(PlanHeader)) {
        acsr_set_error("acsr_plan_status: plan workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    int32_t ovf = 0;
    cudaError_t e = cudaMemcpyAsync(&ovf, &((const PlanHeader *)plan_ws)->overflow, sizeof(int32_t),
                                    cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_plan_status: %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    if (ovf) {
        acsr_set_error("acsr_plan_status: the plan's work list overflowed its workspace (nnz_max passed to "
                       "acsr_bin is smaller than the stored entries); SpMV outputs of this plan are NaN");
        return ACSR_ERR_CAPACITY;
    }
    return ACSR_OK;
}

#if ACSR_TIMELINE
// copies {g_tl (TL_MAX x 2), g_tl_cta (1024 x 3)} to out (TL_MAX*2 + 3072 words), then zeroes them
extern "C" int acsr_debug_timeline(unsigned long long *out)
{
    cudaDeviceSynchronize();
    cudaMemcpyFromSymbol(out, acsr::g_tl, sizeof(acsr::g_tl));
    cudaMemcpyFromSymbol(out + 2 * acsr::TL_MAX, acsr::g_tl_cta, sizeof(acsr::g_tl_cta));
    static unsigned long long z[acsr::TL_MAX][2];
    cudaMemcpyToSymbol(acsr::g_tl, z, sizeof(z));
    return acsr::TL_MAX;
}
#endif

#if ACSR_PROF
extern "C" int acsr_debug_prof(unsigned long long *out16, int reset)
{
    cudaDeviceSynchronize();
    cudaMemcpyFromSymbol(out16, acsr::g_prof, sizeof(unsigned long long) * 16);
    if (reset) {
        unsigned long long z[16] = {0};
        cudaMemcpyToSymbol(acsr::g_prof, z, sizeof(z));
    }
    return 16;
}
#endif
