// acsr_bin.cu -- row binning (Alg. 1 first-iteration preprocessing) and
// the SpMV work map that replaces the G1/G2 split + dynamic parallelism.
//
// Three launches, no host synchronisation:
//   1. bin_count   one CTA per TILE_ROWS-row tile: per-tile histogram of bin ids
//                  (row lengths from the row offsets, P:47 / P:360 "scanning of
//                  row-lengths"), plus per-tile light-unit and heavy-chunk counts.
//   2. bin_scan    one CTA per scan row (32 bins + 2 unit rows): exclusive scan
//                  over tiles; the last CTA turns the bin totals into
//                  bin_offsets[0..32] and the unit totals into the plan header.
//   3. bin_scatter one CTA per tile: stable ranks (warp __match_any_sync + per-warp
//                  counts scanned across warps, 16 rounds of 256 rows in row
//                  order) -> bin_rows; then writes the tile's work units.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdlib.h>

#include "acsr_internal.cuh"

namespace acsr {

namespace cg = cooperative_groups;

template <bool HAS_END>
__device__ __forceinline__ int row_length(const int32_t *__restrict__ rb,
                                          const int32_t *__restrict__ re, int64_t r)
{
    int b = __ldg(rb + r);
    int e = HAS_END ? __ldg(re + r) : __ldg(rb + r + 1);
    return e - b;
}

// Shared scratch of the binning phases (one union per CTA; the fused kernel runs the
// phases back to back in the same CTA).
struct BinSmem {
    // count
    int hist[NBINS];
    int heavy;
    // scan
    int warp_sums[32];
    int carry;
    int is_last;
    // scatter
    int run[NBINS];
    int wcnt[BIN_THREADS / 32][NBINS];
    int wbase[BIN_THREADS / 32][NBINS];
    int seg[NBINS];
    int hw[BIN_THREADS / 32];
    int heavy_run;
    int upre[LIGHT_MAX_BIN + 2];
    int boff[NBINS + 1];  // bin offsets as this CTA sees them (scatter)
    int ovf, nheavy;
};

// ---- phase 1: per-tile histogram of bin ids (+ light-unit / heavy-chunk counts)
template <bool HAS_END>
__device__ __forceinline__ void count_tile(BinSmem &sm, int64_t n, const int32_t *__restrict__ rb,
                                           const int32_t *__restrict__ re, int32_t *__restrict__ cnt,
                                           int n_tiles, int tile, int wmb)
{
    const int tid = threadIdx.x;
    if (tid < NBINS) sm.hist[tid] = 0;
    if (tid == 0) sm.heavy = 0;
    __syncthreads();
    const int64_t base = (int64_t)tile * TILE_ROWS;
    int my_heavy = 0;
    int lens[TILE_ROUNDS];
#pragma unroll
    for (int k = 0; k < TILE_ROUNDS; k++) {  // all row-length loads in flight at once
        const int64_t r = base + k * BIN_THREADS + tid;
        lens[k] = r < n ? row_length<HAS_END>(rb, re, r) : -1;
    }
#pragma unroll
    for (int k = 0; k < TILE_ROUNDS; k++) {
        const bool valid = lens[k] >= 0;
        const int len = valid ? lens[k] : 0;
        const int b = valid ? bin_of_len(len) : NBINS;
        // warp-aggregated histogram update: one shared atomic per distinct bin
        const unsigned m = __match_any_sync(0xffffffffu, b);
        if (valid && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&sm.hist[b], __popc(m));
        if (b >= HEAVY_BIN && valid) my_heavy += heavy_chunks(len);
    }
    for (int o = 16; o > 0; o >>= 1) my_heavy += __shfl_xor_sync(0xffffffffu, my_heavy, o);
    if ((tid & 31) == 0 && my_heavy) atomicAdd(&sm.heavy, my_heavy);
    __syncthreads();
    if (tid < 32) {  // warp 0: the tile's row of counts; light units one bin per lane, summed
        static_assert(NBINS == 32, "one lane per bin");
        const int h = sm.hist[tid];
        cnt[(int64_t)tid * n_tiles + tile] = h;
        const bool tl = tail_tile(tile, n_tiles);
        int lu = 0;
        if (tid > wmb && tid <= LIGHT_MAX_BIN) lu = ceil_shift(h, unit_shift_t(tid, tl));
        lu = __reduce_add_sync(0xffffffffu, lu);
        if (tid == 0) {
            if (wmb >= 0) lu += win_units_t((int)min((int64_t)TILE_ROWS, n - base), tl);
            cnt[(int64_t)NBINS * n_tiles + tile] = lu;
            cnt[(int64_t)(NBINS + 1) * n_tiles + tile] = sm.heavy;
        }
    }
    __syncthreads();
}

struct ScanArgs {
    int32_t *bin_offsets;
    int64_t n_cols, light_cap, heavy_cap;
    PlanLayout L;
    int xc_valid, xc_stride;
};

// ---- phase 2: exclusive scan of one scan row over the tiles (coalesced chunks of T
// with a running carry); the last of the SCAN_ROWS rows to finish turns the totals
// into bin_offsets and the plan header.
template <int T, int IPT, bool FINALIZE = true>
__device__ __forceinline__ void scan_row(BinSmem &sm, const int32_t *__restrict__ cnt,
                                         int32_t *__restrict__ toff, int n_tiles, PlanHeader *hdr,
                                         const ScanArgs &sa, int row)
{
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int32_t *a = cnt + (int64_t)row * n_tiles;
    int32_t *o = toff + (int64_t)row * n_tiles;
    if (tid == 0) sm.carry = 0;
    __syncthreads();
    // chunks of T * IPT elements; thread t owns IPT consecutive elements of a chunk
    for (int c0 = 0; c0 < n_tiles; c0 += T * IPT) {
        const int i0 = c0 + tid * IPT;
        int v[IPT];
        int s = 0;
#pragma unroll
        for (int j = 0; j < IPT; j++) {
            v[j] = i0 + j < n_tiles ? a[i0 + j] : 0;
            s += v[j];
        }
        int incl = s;
        for (int d = 1; d < 32; d <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += t;
        }
        if (lane == 31) sm.warp_sums[warp] = incl;
        __syncthreads();
        if (warp == 0) {
            const int w = lane < T / 32 ? sm.warp_sums[lane] : 0;
            int wi = w;
            for (int d = 1; d < 32; d <<= 1) {
                const int t = __shfl_up_sync(0xffffffffu, wi, d);
                if (lane >= d) wi += t;
            }
            if (lane < T / 32) sm.warp_sums[lane] = wi - w;  // exclusive
        }
        __syncthreads();
        const int base_c = sm.carry;
        int run = base_c + sm.warp_sums[warp] + incl - s;
#pragma unroll
        for (int j = 0; j < IPT; j++) {
            if (i0 + j < n_tiles) o[i0 + j] = run;
            run += v[j];
        }
        __syncthreads();
        if (tid == T - 1) sm.carry = run;
        __syncthreads();
    }
    if (tid == 0) hdr->totals[row] = sm.carry;
    __syncthreads();
    if (!FINALIZE) return;  // the scatter kernel turns the totals into offsets + header
    if (tid == 0) {
        __threadfence();
        sm.is_last = (atomicAdd(&hdr->scan_ticket, 1) == SCAN_ROWS - 1);
    }
    __syncthreads();
    if (sm.is_last && warp == 0) {
        // one parallel load per lane (not a serial chain of L2 round trips)
        __threadfence();
        const int t = __ldcg(hdr->totals + lane);
        int incl = t;
        for (int d = 1; d < 32; d <<= 1) {
            const int v = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += v;
        }
        sa.bin_offsets[lane] = incl - t;
        if (lane == 31) sa.bin_offsets[NBINS] = incl;  // == n_rows
    }
    if (sm.is_last && tid == 0) {
        const int nl = __ldcg(hdr->totals + NBINS), nh = __ldcg(hdr->totals + NBINS + 1);
        const int ovf = (nl > sa.light_cap) || (nh > sa.heavy_cap);
        hdr->overflow = ovf;
        hdr->n_light_units = ovf ? 0 : nl;
        hdr->n_heavy_units = ovf ? 0 : nh;
        hdr->n_units = ovf ? 0 : nl + nh;
        hdr->n_tiles = n_tiles;
        hdr->off_units = (int64_t)sa.L.off_units;
        hdr->off_partial = (int64_t)sa.L.off_partial;
        hdr->off_ticket = (int64_t)sa.L.off_ticket;
        hdr->off_xc_vote = (int64_t)sa.L.off_xc_vote;
        hdr->off_xc_tag = (int64_t)sa.L.off_xc_tag;
        hdr->off_xc_val = (int64_t)sa.L.off_xc_val;
        hdr->off_tile_done = (int64_t)sa.L.off_tile_done;
        hdr->xc_valid = sa.xc_valid;
        hdr->xc_stride = sa.xc_stride;
        hdr->n_cols = sa.n_cols;
        hdr->work_ctr = 0;
        hdr->exit_ticket = 0;
        hdr->d2_hi = 0;
        hdr->d2_mid = 0;
        hdr->d2_lo = 0;
        hdr->scan_ticket = 0;
    }
    __syncthreads();
}

// Scatter prologue, default path (warp 0): the 34 scan-row totals -> bin offsets (warp
// scan), overflow and heavy-unit count, in shared memory; block 0 also publishes
// bin_offsets and the plan header the SpMV reads.  Replaces the scan kernel's
// last-CTA finalisation (ticket -> totals -> offsets: a chain of dependent L2 round trips).
__device__ __forceinline__ void plan_from_totals(BinSmem &sm, PlanHeader *hdr, const ScanArgs &sa, int n_tiles,
                                                 bool publish)
{
    const int lane = threadIdx.x & 31;
    if (threadIdx.x >= 32) return;
    const int t = __ldcg(hdr->totals + lane);  // NBINS == 32 == warp size
    int incl = t;
    for (int d = 1; d < 32; d <<= 1) {
        const int v = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += v;
    }
    sm.boff[lane] = incl - t;
    if (lane == 31) sm.boff[NBINS] = incl;
    const int nl = __ldcg(hdr->totals + NBINS), nh = __ldcg(hdr->totals + NBINS + 1);
    const int ovf = (nl > sa.light_cap) || (nh > sa.heavy_cap);
    if (lane == 0) {
        sm.ovf = ovf;
        sm.nheavy = ovf ? 0 : nh;
    }
    if (!publish) return;
    sa.bin_offsets[lane] = incl - t;
    if (lane == 31) sa.bin_offsets[NBINS] = incl;  // == n_rows
    if (lane == 0) {
        hdr->overflow = ovf;
        hdr->n_light_units = ovf ? 0 : nl;
        hdr->n_heavy_units = ovf ? 0 : nh;
        hdr->n_units = ovf ? 0 : nl + nh;
        hdr->n_tiles = n_tiles;
        hdr->off_units = (int64_t)sa.L.off_units;
        hdr->off_partial = (int64_t)sa.L.off_partial;
        hdr->off_ticket = (int64_t)sa.L.off_ticket;
        hdr->off_xc_vote = (int64_t)sa.L.off_xc_vote;
        hdr->off_xc_tag = (int64_t)sa.L.off_xc_tag;
        hdr->off_xc_val = (int64_t)sa.L.off_xc_val;
        hdr->off_tile_done = (int64_t)sa.L.off_tile_done;
        hdr->xc_valid = sa.xc_valid;
        hdr->xc_stride = sa.xc_stride;
        hdr->n_cols = sa.n_cols;
        hdr->work_ctr = 0;
        hdr->exit_ticket = 0;
        hdr->d2_hi = 0;
        hdr->d2_mid = 0;
        hdr->d2_lo = 0;
    }
}

// Scatter prologue of the fused paths: offsets and header were published by the
// finalising scan CTA of the same grid (coherent L2 loads)
__device__ __forceinline__ void plan_from_global(BinSmem &sm, const PlanHeader *hdr, const int32_t *bin_offsets)
{
    const int tid = threadIdx.x;
    if (tid <= NBINS) sm.boff[tid] = __ldcg(bin_offsets + tid);
    if (tid == 0) {
        sm.ovf = __ldcg(&hdr->overflow);
        sm.nheavy = __ldcg(&hdr->n_heavy_units);
    }
}

// ---- phase 3: stable scatter of one tile + its work units
// The tile's inputs that do not depend on the plan (row lengths, the tile's row of the
// per-tile prefixes) are loaded first, so their latency overlaps the plan prologue.
struct ScatterPre {
    int lens[TILE_ROUNDS];
    int tof;   // toff[tid][tile] (tid < NBINS)
    int hrun;  // toff[heavy row][tile] (tid == 0)
    int lu;    // toff[light-unit row][tile] (every thread)
};

template <bool HAS_END>
__device__ __forceinline__ void scatter_preload(ScatterPre &pre, int64_t n, const int32_t *__restrict__ rb,
                                                const int32_t *__restrict__ re, const int32_t *toff, int n_tiles,
                                                int tile)
{
    const int tid = threadIdx.x;
    const int64_t base = (int64_t)tile * TILE_ROWS;
#pragma unroll
    for (int k = 0; k < TILE_ROUNDS; k++) {  // all row-length loads in flight at once
        const int64_t r = base + k * BIN_THREADS + tid;
        pre.lens[k] = r < n ? row_length<HAS_END>(rb, re, r) : 0;
    }
    pre.tof = tid < NBINS ? __ldcg(toff + (int64_t)tid * n_tiles + tile) : 0;
    pre.hrun = tid == 0 ? __ldcg(toff + (int64_t)(NBINS + 1) * n_tiles + tile) : 0;
    pre.lu = __ldcg(toff + (int64_t)NBINS * n_tiles + tile);
}

template <bool HAS_END>
__device__ __forceinline__ void scatter_tile(BinSmem &sm, const ScatterPre &pre, int64_t n,
                                             int32_t *__restrict__ bin_rows, int n_tiles,
                                             int2 *__restrict__ units, int32_t *__restrict__ tickets,
                                             int64_t heavy_cap, int tile, int wmb, int32_t *tile_done)
{
    if (threadIdx.x == 0) tile_done[tile] = 0;  // the fused peer exchange's per-tile row count
    constexpr int NW = BIN_THREADS / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // sm.boff / sm.ovf / sm.nheavy were filled by the caller (plan_from_totals or
    // plan_from_global) before a __syncthreads
    const int overflow = sm.ovf;
    const int n_heavy = sm.nheavy;
    if (tid < NBINS) {
        sm.run[tid] = 0;
        sm.seg[tid] = sm.boff[tid] + pre.tof;
    }
    for (int i = tid; i < NW * NBINS; i += BIN_THREADS) (&sm.wcnt[0][0])[i] = 0;
    if (tid == 0) sm.heavy_run = pre.hrun;
    __syncthreads();
    const int64_t base = (int64_t)tile * TILE_ROWS;
    const unsigned lt = (1u << lane) - 1u;
    int lens[TILE_ROUNDS];
#pragma unroll
    for (int k = 0; k < TILE_ROUNDS; k++) lens[k] = pre.lens[k];
#pragma unroll
    for (int k = 0; k < TILE_ROUNDS; k++) {
        const int64_t r = base + k * BIN_THREADS + tid;
        const bool valid = r < n;
        const int len = lens[k];
        const int b = valid ? bin_of_len(len) : NBINS;  // NBINS = sentinel for past-the-end rows
        const unsigned mask = __match_any_sync(0xffffffffu, b);
        const int rank = __popc(mask & lt);
        if (valid && rank == 0) sm.wcnt[warp][b] = __popc(mask);
        const int hc = (valid && b >= HEAVY_BIN) ? heavy_chunks(len) : 0;
        int hincl = hc;
        for (int d = 1; d < 32; d <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, hincl, d);
            if (lane >= d) hincl += t;
        }
        if (lane == 31) sm.hw[warp] = hincl;
        __syncthreads();
        if (tid < NBINS) {
            int acc = sm.run[tid];
#pragma unroll
            for (int w = 0; w < NW; w++) {
                sm.wbase[w][tid] = acc;
                acc += sm.wcnt[w][tid];
                sm.wcnt[w][tid] = 0;
            }
            sm.run[tid] = acc;
        } else if (tid == NBINS) {
            int acc = sm.heavy_run;
#pragma unroll
            for (int w = 0; w < NW; w++) {
                const int t = sm.hw[w];
                sm.hw[w] = acc;
                acc += t;
            }
            sm.heavy_run = acc;
        }
        __syncthreads();
        if (valid) {
            bin_rows[sm.seg[b] + sm.wbase[warp][b] + rank] = (int32_t)r;
            if (hc > 0 && !overflow) {
                const int u0 = sm.hw[warp] + hincl - hc;
                for (int c = 0; c < hc; c++)
                    if (u0 + c < heavy_cap) units[u0 + c] = make_int2((int)r, (int)(HEAVY_FLAG | (uint32_t)c));
                if (u0 < heavy_cap) tickets[u0] = 0;
            }
        }
        __syncthreads();
    }
    if (!overflow) {
        // light work units of this tile: the short-row windows (row order), then the
        // bins above wmb up to 10, in bin order, row-contiguous (wmb = -1: no windows,
        // bins 0..10 as per-bin units -- Alg. 2 for the short bins)
        const int tile_rows = (int)min((int64_t)TILE_ROWS, n - base);
        const bool tl = tail_tile(tile, n_tiles);
        const int wur = win_unit_rows_t(tl);
        const int nwin = wmb >= 0 ? win_units_t(tile_rows, tl) : 0;
        if (tid == 0) {
            int acc = nwin;
            for (int b = 0; b <= LIGHT_MAX_BIN; b++) {
                sm.upre[b] = acc;
                if (b > wmb) acc += ceil_shift(sm.run[b], unit_shift_t(b, tl));
            }
            sm.upre[LIGHT_MAX_BIN + 1] = acc;
        }
        __syncthreads();
        const int ubase = n_heavy + pre.lu;
        const int total = sm.upre[LIGHT_MAX_BIN + 1];
        for (int j = tid; j < total; j += BIN_THREADS) {
            if (j < nwin) {
                const int r0 = j * wur;
                units[ubase + j] = make_int2((int)(base + r0), (int)(WIN_FLAG | (uint32_t)min(wur, tile_rows - r0)));
                continue;
            }
            int b = 0;
            while (sm.upre[b + 1] <= j) b++;
            const int q = j - sm.upre[b];
            const int K = unit_rows_t(b, tl);
            const int c = min(K, sm.run[b] - q * K);
            units[ubase + j] = make_int2(sm.seg[b] + q * K, (b << 24) | c);
        }
    }
    __syncthreads();
}

// ---- three-launch path (used when a cooperative launch is not possible)
template <bool HAS_END>
__global__ void __launch_bounds__(BIN_THREADS, 2048 / BIN_THREADS)
bin_count_kernel(int64_t n, const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                 int32_t *__restrict__ cnt, int n_tiles, PlanHeader *hdr, int wmb)
{
    __shared__ BinSmem sm;
    pdl_enter();
    if (blockIdx.x == 0 && threadIdx.x == 0) {  // the scan (or fused scan+scatter) launch runs after us
        hdr->scan_ticket = 0;
        hdr->role_ticket = 0;
        hdr->scan_done = 0;
    }
    count_tile<HAS_END>(sm, n, rb, re, cnt, n_tiles, blockIdx.x, wmb);
}

#ifndef ACSR_SCAN_THREADS
#define ACSR_SCAN_THREADS 1024  // A/B: 256 with 4 values per thread
#endif
constexpr int SCAN_THREADS = ACSR_SCAN_THREADS;
constexpr int SCAN_IPT = SCAN_THREADS >= 1024 ? 1 : 1024 / SCAN_THREADS;

__global__ void __launch_bounds__(SCAN_THREADS)
bin_scan_kernel(const int32_t *__restrict__ cnt, int32_t *__restrict__ toff, int n_tiles,
                PlanHeader *hdr, ScanArgs sa)
{
    __shared__ BinSmem sm;
    pdl_enter();
    scan_row<SCAN_THREADS, SCAN_IPT, false>(sm, cnt, toff, n_tiles, hdr, sa, blockIdx.x);
}

template <bool HAS_END>
__global__ void __launch_bounds__(BIN_THREADS, 2048 / BIN_THREADS)
bin_scatter_kernel(int64_t n, const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                   int32_t *__restrict__ bin_rows, const int32_t *__restrict__ toff, int n_tiles,
                   PlanHeader *hdr, int2 *__restrict__ units, int32_t *__restrict__ tickets, ScanArgs sa,
                   int wmb)
{
    __shared__ BinSmem sm;
    pdl_enter();
    ScatterPre pre;
    scatter_preload<HAS_END>(pre, n, rb, re, toff, n_tiles, blockIdx.x);  // overlaps the prologue
    plan_from_totals(sm, hdr, sa, n_tiles, blockIdx.x == 0);
    __syncthreads();
    scatter_tile<HAS_END>(sm, pre, n, bin_rows, n_tiles, units, tickets, sa.heavy_cap, blockIdx.x, wmb,
                          (int32_t *)((char *)hdr + sa.L.off_tile_done));
}

// ---- scan + scatter in ONE launch (opt-in, ACSR_BIN_SS=1): the first SCAN_ROWS CTAs to start (an
// atomic role ticket, reset by bin_count) scan one row each -- the last of them writes
// bin_offsets and the plan header -- and count themselves done; every other CTA takes a
// tile, prefetches the tile's row offsets into L2, waits until all scan rows are done and
// scatters.  The scanning CTAs are already running when anyone waits (they took the
// first tickets), so the wait cannot deadlock.  Saves the scan kernel's launch boundary
// but measured slower (see scan_scatter_fused).
template <bool HAS_END>
__global__ void __launch_bounds__(BIN_THREADS, 2048 / BIN_THREADS)
bin_scan_scatter_kernel(int64_t n, const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                        const int32_t *__restrict__ cnt, int32_t *__restrict__ toff, int32_t *__restrict__ bin_rows,
                        int n_tiles, PlanHeader *hdr, ScanArgs sa, int2 *__restrict__ units,
                        int32_t *__restrict__ tickets, int wmb)
{
    __shared__ BinSmem sm;
    __shared__ int s_role;
    pdl_enter();
    if (threadIdx.x == 0) s_role = atomicAdd(&hdr->role_ticket, 1);
    __syncthreads();
    const int role = s_role;
    if (role < SCAN_ROWS) {
        scan_row<BIN_THREADS, 8>(sm, cnt, toff, n_tiles, hdr, sa, role);
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(&hdr->scan_done, 1);
        }
        return;
    }
    const int tile = role - SCAN_ROWS;
    {
        const int64_t base = (int64_t)tile * TILE_ROWS;
        const int64_t rows = min((int64_t)TILE_ROWS + 1, n + 1 - base);
        const int64_t off = (int64_t)threadIdx.x * 32;  // 128-byte lines of the tile's offsets
        if (off < rows) asm volatile("prefetch.global.L2 [%0];" ::"l"(rb + base + off));
        if (HAS_END && off < rows - 1) asm volatile("prefetch.global.L2 [%0];" ::"l"(re + base + off));
    }
    if (threadIdx.x == 0)
        while (*(volatile int32_t *)&hdr->scan_done < SCAN_ROWS) __nanosleep(64);
    __syncthreads();
    __threadfence();
    plan_from_global(sm, hdr, sa.bin_offsets);
    ScatterPre pre;
    scatter_preload<HAS_END>(pre, n, rb, re, toff, n_tiles, tile);  // toff is complete after the wait
    __syncthreads();
    scatter_tile<HAS_END>(sm, pre, n, bin_rows, n_tiles, units, tickets, sa.heavy_cap, tile, wmb,
                          (int32_t *)((char *)hdr + sa.L.off_tile_done));
}

// ---- one cooperative launch: count -> grid barrier -> scan -> grid barrier -> scatter
// (two grid-wide barriers instead of two kernel boundaries; tiles are grid-strided)
struct FusedArgs {
    int64_t n;
    const int32_t *rb, *re;
    int32_t *cnt, *toff, *bin_rows, *tickets;
    int2 *units;
    PlanHeader *hdr;
    int n_tiles;
    ScanArgs sa;
    int wmb;
};

template <bool HAS_END>
__global__ void __launch_bounds__(BIN_THREADS, 2048 / BIN_THREADS)
bin_fused_kernel(FusedArgs f)
{
    __shared__ BinSmem sm;
    cg::grid_group grid = cg::this_grid();
    if (blockIdx.x == 0 && threadIdx.x == 0) f.hdr->scan_ticket = 0;
    for (int t = blockIdx.x; t < f.n_tiles; t += gridDim.x)
        count_tile<HAS_END>(sm, f.n, f.rb, f.re, f.cnt, f.n_tiles, t, f.wmb);
    grid.sync();
    for (int row = blockIdx.x; row < SCAN_ROWS; row += gridDim.x)
        scan_row<BIN_THREADS, 8>(sm, f.cnt, f.toff, f.n_tiles, f.hdr, f.sa, row);
    grid.sync();
    plan_from_global(sm, f.hdr, f.sa.bin_offsets);
    __syncthreads();
    for (int t = blockIdx.x; t < f.n_tiles; t += gridDim.x) {
        ScatterPre pre;
        scatter_preload<HAS_END>(pre, f.n, f.rb, f.re, f.toff, f.n_tiles, t);
        scatter_tile<HAS_END>(sm, pre, f.n, f.bin_rows, f.n_tiles, f.units,
                              f.tickets, f.sa.heavy_cap, t, f.wmb, (int32_t *)((char *)f.hdr + f.sa.L.off_tile_done));
    }
}

// x-cache table: sampled occurrence counts, per-slot winner (count, column).
__global__ void xc_count_kernel(const int32_t *__restrict__ col, int64_t nnz_max, int64_t n_cols,
                                int stride, int32_t *__restrict__ count,
                                unsigned long long *__restrict__ best)
{
    const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t k = j * stride + (int64_t)(mix32((uint32_t)j) % (uint32_t)stride);
    if (k >= nnz_max) return;
    const int c = __ldg(col + k);
    if (c < 0 || c >= n_cols) return;  // slack entries / garbage: a hint only
    const int cnt = atomicAdd(count + c, 1) + 1;
    atomicMax(best + (c & (XC_SLOTS - 1)), ((unsigned long long)cnt << 32) | (unsigned)c);
}

}  // namespace acsr

using namespace acsr;

// ACSR_BIN_FUSED=1 selects the single cooperative launch.  Measured slower on B200
// (C2: 28.7 vs 25.6 us; LiveJournal-like: 65.5 vs 48.1 us; s26: 0.87 vs 0.61 ms -- the
// grid-wide syncs and the cooperative launch cost more than the two kernel boundaries
// they replace), so the three-launch path is the default.
static bool fused_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("ACSR_BIN_FUSED");
        v = (e && e[0] == '1') ? 1 : 0;
    }
    return v == 1;
}

// ACSR_BIN_SS=1 selects the fused scan+scatter launch.  Measured slower on B200 (C2 bin
// 27.6 vs 25.6 us, LiveJournal-like 93 vs 52 us, s26 1.30 vs 0.64 ms: the 34 scan rows on
// 256-thread CTAs serialise in front of every waiting scatter CTA), so the separate scan
// kernel is the default.
static bool scan_scatter_fused()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("ACSR_BIN_SS");
        v = (e && e[0] == '1') ? 1 : 0;
    }
    return v == 1;
}

static int fused_grid(bool has_end)
{
    static int g[2] = {0, 0};
    int &gg = g[has_end ? 1 : 0];
    if (!gg) {
        int per_sm = 0;
        if (has_end)
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bin_fused_kernel<true>, BIN_THREADS, 0);
        else
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bin_fused_kernel<false>, BIN_THREADS, 0);
        if (per_sm < 1) per_sm = 1;
        gg = per_sm * acsr_num_sms();
    }
    return gg;
}

extern "C" size_t acsr_bin_workspace_bytes(int64_t n_rows, int64_t n_cols, int64_t nnz_max)
{
    if (n_rows < 0 || n_cols < 0 || nnz_max < 0) return 0;
    return plan_layout(n_rows, n_cols, nnz_max).total;
}

extern "C" acsr_status acsr_bin_ex(int64_t n_rows, int64_t n_cols, int64_t nnz_max,
                                   const int32_t *row_begin, const int32_t *row_end,
                                   const int32_t *col_idx, int32_t *bin_rows, int32_t *bin_offsets,
                                   void *plan_ws, size_t plan_ws_bytes, unsigned flags, cudaStream_t stream)
{
    if ((flags & ~(unsigned)ACSR_BIN_SHORT_ALG2) != 0) {
        acsr_set_error("acsr_bin_ex: unknown flags 0x%x", flags);
        return ACSR_ERR_INVALID_VALUE;
    }
    const int wmb = (flags & ACSR_BIN_SHORT_ALG2) ? -1 : WIN_MAX_BIN;
    if (n_rows < 0 || n_cols < 0 || nnz_max < 0 || n_rows >= (int64_t)1 << 31 || !bin_offsets ||
        (n_rows > 0 && (!row_begin || !bin_rows))) {
        acsr_set_error("acsr_bin: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    PlanLayout L = plan_layout(n_rows, n_cols, nnz_max);
    if (!plan_ws || plan_ws_bytes < L.total) {
        acsr_set_error("acsr_bin: workspace %zu < required %zu", plan_ws_bytes, L.total);
        return ACSR_ERR_WORKSPACE;
    }
    char *ws = (char *)plan_ws;
    PlanHeader *hdr = (PlanHeader *)ws;
    if (n_rows == 0) {
        cudaMemsetAsync(hdr, 0, sizeof(PlanHeader), stream);
        cudaMemsetAsync(bin_offsets, 0, sizeof(int32_t) * (NBINS + 1), stream);
        return acsr_check_launch("acsr_bin(empty)");
    }
    int32_t *cnt = (int32_t *)(ws + L.off_cnt);
    int32_t *toff = (int32_t *)(ws + L.off_toff);
    int2 *units = (int2 *)(ws + L.off_units);
    int32_t *tickets = (int32_t *)(ws + L.off_ticket);
    const int nt = (int)L.n_tiles;
    // the x-cache table is built only when the (experimental, default-off) cache is enabled
    const char *xe = getenv("ACSR_XCACHE");
    const int xc_valid = xe && xe[0] == '1' && col_idx != nullptr && n_cols > 0 &&
                         n_cols < ((int64_t)XC_NOTAG << XC_BITS);
    int64_t stride64 = nnz_max >> XC_SAMPLE_LOG2;
    const int xc_stride = (int)(stride64 < 1 ? 1 : (stride64 > (1 << 30) ? (1 << 30) : stride64));
    ScanArgs sa{bin_offsets, n_cols, L.light_cap, L.heavy_cap, L, xc_valid, xc_stride};
    if (fused_enabled()) {
        FusedArgs f{n_rows, row_begin, row_end, cnt, toff, bin_rows, tickets, units, hdr, nt, sa, wmb};
        const int grid = fused_grid(row_end != nullptr);
        void *args[] = {&f};
        const cudaError_t e = row_end
            ? cudaLaunchCooperativeKernel((void *)bin_fused_kernel<true>, grid, BIN_THREADS, args, 0, stream)
            : cudaLaunchCooperativeKernel((void *)bin_fused_kernel<false>, grid, BIN_THREADS, args, 0, stream);
        if (e == cudaSuccess) goto xc;
        cudaGetLastError();  // not supported here (e.g. MPS limits): fall back to three launches
    }
    {
        const int64_t nr = n_rows;
        const int32_t *rb = row_begin, *re = row_end;
        const int32_t *ctoff = toff;
        if (row_end)
            launch_pdl(bin_count_kernel<true>, nt, BIN_THREADS, 0, stream, nr, rb, re, cnt, nt, hdr, wmb);
        else
            launch_pdl(bin_count_kernel<false>, nt, BIN_THREADS, 0, stream, nr, rb, re, cnt, nt, hdr, wmb);
        const int32_t *ccnt = cnt;
        if (scan_scatter_fused()) {
            if (row_end)
                launch_pdl(bin_scan_scatter_kernel<true>, nt + SCAN_ROWS, BIN_THREADS, 0, stream, nr, rb, re, ccnt,
                           toff, bin_rows, nt, hdr, sa, units, tickets, wmb);
            else
                launch_pdl(bin_scan_scatter_kernel<false>, nt + SCAN_ROWS, BIN_THREADS, 0, stream, nr, rb, re, ccnt,
                           toff, bin_rows, nt, hdr, sa, units, tickets, wmb);
            goto xc;
        }
        launch_pdl(bin_scan_kernel, SCAN_ROWS, SCAN_THREADS, 0, stream, ccnt, toff, nt, hdr, sa);
        if (row_end)
            launch_pdl(bin_scatter_kernel<true>, nt, BIN_THREADS, 0, stream, nr, rb, re, bin_rows, ctoff, nt, hdr,
                       units, tickets, sa, wmb);
        else
            launch_pdl(bin_scatter_kernel<false>, nt, BIN_THREADS, 0, stream, nr, rb, re, bin_rows, ctoff, nt, hdr,
                       units, tickets, sa, wmb);
    }
xc:
    if (xc_valid) {
        cudaMemsetAsync(ws + L.off_xc_vote, 0, sizeof(uint64_t) * XC_SLOTS, stream);
        cudaMemsetAsync(ws + L.off_xc_count, 0, sizeof(int32_t) * (size_t)n_cols, stream);
        const int64_t samples = (nnz_max + xc_stride - 1) / xc_stride;
        xc_count_kernel<<<(unsigned)((samples + 255) / 256), 256, 0, stream>>>(
            col_idx, nnz_max, n_cols, xc_stride, (int32_t *)(ws + L.off_xc_count),
            (unsigned long long *)(ws + L.off_xc_vote));
    }
    return acsr_check_launch("acsr_bin");
}

extern "C" acsr_status acsr_bin(int64_t n_rows, int64_t n_cols, int64_t nnz_max,
                                const int32_t *row_begin, const int32_t *row_end,
                                const int32_t *col_idx, int32_t *bin_rows, int32_t *bin_offsets,
                                void *plan_ws, size_t plan_ws_bytes, cudaStream_t stream)
{
    return acsr_bin_ex(n_rows, n_cols, nnz_max, row_begin, row_end, col_idx, bin_rows, bin_offsets, plan_ws,
                       plan_ws_bytes, 0u, stream);
}
