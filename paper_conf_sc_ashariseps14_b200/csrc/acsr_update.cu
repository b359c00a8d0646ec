// acsr_update.cu -- dynamic-graph update on slack CSR (§VII).
//
// The paper uses one warp per updated row with only its first thread working
// (P:335).  Here every lane works: pass 1 validates the whole batch (one warp per
// update, deletes counted by binary search in the sorted delete list) and records
// the smallest failing index with a 64-bit atomicMin; pass 2 (only if the batch is
// valid -- all-or-nothing, reading Q13) compacts each row with a warp ballot
// prefix (stable, in place: a lane's destination is never past its source) and
// appends the inserts lane-parallel.  Out-degrees change by integer atomics, so
// the result is exact and independent of scheduling.
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>

#include "acsr_internal.cuh"

namespace acsr {

constexpr int UPD_THREADS = 256;
constexpr unsigned long long NO_FAIL = ~0ull;
// rows longer than this with a non-empty delete list are validated and compacted by a
// whole CTA (block-scan compaction) instead of one warp: hub rows of power-law graphs
constexpr int LONG_ROW = 2048;

struct UpdWs {
    unsigned long long key;  // (first failing index << 3) | code, or NO_FAIL
    unsigned int n_long;     // number of long-row updates appended to long_list
    unsigned int pad;
    long long n_eff;         // updates of this batch (host count, or the device count of
                             // acsr_update_edges_dev), written by update_init_kernel
    int32_t long_list[1];    // [n_upd]
};

// hub rows: the delete list is staged in shared memory when it has at most del_cap entries
// (dynamic shared memory, up to DEL_SMEM_MAX ints = 192 KB) and binary-searched there
constexpr int DEL_SMEM_MAX = 48 * 1024;

__device__ __forceinline__ bool member_s(const int32_t *d, int m, int c)
{
    int l = 0, h = m;
    while (l < h) {
        int mid = (l + h) >> 1;
        if (d[mid] < c) l = mid + 1;
        else h = mid;
    }
    return l < m && d[l] == c;
}

// short delete lists (<= 32 entries): lane t holds entry t in a register and membership is
// tested with m warp shuffles instead of a dependent binary search in global memory
// (called by all 32 lanes with the same m)
__device__ __forceinline__ bool member_w(int dreg, int m, int c)
{
    bool hit = false;
    for (int j = 0; j < m; j++) hit |= __shfl_sync(0xffffffffu, dreg, j) == c;
    return hit;
}

#ifndef ACSR_UPD_WARPREG
#define ACSR_UPD_WARPREG 0  // 1: register/shuffle membership for <= 32 deletes (A/B: neutral on N2)
#endif

__device__ __forceinline__ bool member(const int32_t *__restrict__ d, int lo, int hi, int c)
{
    int l = lo, h = hi;
    while (l < h) {
        int mid = (l + h) >> 1;
        if (__ldg(d + mid) < c) l = mid + 1;
        else h = mid;
    }
    return l < hi && __ldg(d + l) == c;
}

// validation of update i by one full warp (called warp-uniformly)
__device__ __forceinline__ void validate_row(int64_t i, int lane, int64_t n_rows, int64_t n_cols,
                                             const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                                             const int32_t *__restrict__ cap, const int32_t *__restrict__ col,
                                             const int32_t *__restrict__ upd, const int32_t *__restrict__ dptr,
                                             const int32_t *__restrict__ dcol, const int32_t *__restrict__ iptr,
                                             const int32_t *__restrict__ icol, UpdWs *ws)
{
    unsigned long long *key = &ws->key;
    // every load that does not depend on another is issued first (row id, previous row id,
    // list bounds, then the row's bounds and capacity): the checks below overlap them
    // instead of each waiting behind the previous check's warp vote
    const int r = __ldg(upd + i);
    const int rprev = i > 0 ? __ldg(upd + i - 1) : -1;
    const int d0 = dptr ? __ldg(dptr + i) : 0, d1 = dptr ? __ldg(dptr + i + 1) : 0;
    const int i0 = __ldg(iptr + i), i1 = __ldg(iptr + i + 1);
    const bool rok = r >= 0 && r < n_rows;
    const int b = rok ? __ldg(rb + r) : 0, e = rok ? __ldg(re + r) : 0;
    const int cp = rok ? __ldg(cap + r) : 0;
    // checks in reading R1's order: (a) row id, (b) delete list sorted, (c) insert columns
    // in range -- (a)-(c) all give INVALID_VALUE, so one vote covers (b) and (c) -- then (d)
    int code = (!rok || (i > 0 && r <= rprev)) ? ACSR_ERR_INVALID_VALUE : ACSR_OK;
    bool bad = false;
    for (int j = d0 + 1 + lane; j < d1; j += 32) bad |= __ldg(dcol + j) < __ldg(dcol + j - 1);
    for (int j = i0 + lane; j < i1; j += 32) {
        const int c = __ldg(icol + j);
        bad |= (c < 0 || c >= n_cols);
    }
    if (__any_sync(0xffffffffu, bad) && code == ACSR_OK) code = ACSR_ERR_INVALID_VALUE;
    if (code == ACSR_OK) {
        if (d1 > d0 && e - b > LONG_ROW) {  // deferred to the CTA-per-row kernel
            if (lane == 0) ws->long_list[atomicAdd(&ws->n_long, 1u)] = (int32_t)i;
            return;
        }
        int dels = 0;
        const int m = d1 - d0;
        if (ACSR_UPD_WARPREG && m > 0 && m <= 32) {
            const int dreg = lane < m ? __ldg(dcol + d0 + lane) : 0;
            for (int k0 = b; k0 < e; k0 += 32) {  // warp-uniform trip count (shuffles)
                const bool valid = k0 + lane < e;
                const int c = valid ? __ldg(col + k0 + lane) : 0;
                dels += (member_w(dreg, m, c) && valid) ? 1 : 0;
            }
        } else if (m > 0) {
            for (int k = b + lane; k < e; k += 32) dels += member(dcol, d0, d1, __ldg(col + k)) ? 1 : 0;
        }
        for (int o = 16; o > 0; o >>= 1) dels += __shfl_xor_sync(0xffffffffu, dels, o);
        long long new_len = (long long)(e - b) - dels + (i1 - i0);
        if (new_len > cp) code = ACSR_ERR_CAPACITY;
    }
    if (code != ACSR_OK && lane == 0) atomicMin(key, ((unsigned long long)i << 3) | (unsigned)code);
}

// Short rows, four per warp: an 8-lane sub-warp per update (SUB_W lanes, SUB_R = 32/SUB_W
// updates per warp) when every row of the warp has at most SUB_MAX entries -- the
// per-row chain of dependent loads (update -> row bounds -> columns -> delete-list
// search) is latency-bound, so more rows in flight per warp is what pays.  Otherwise
// the warp validates its rows one after another with validate_row.
constexpr int SUB_W = 8, SUB_R = 32 / SUB_W, SUB_MAX = 64;
#ifndef ACSR_UPD_SUB
#define ACSR_UPD_SUB 0  // 1: 8-lane sub-warps for short rows (A/B: N2 update 0.36 -> 0.45 ms, slower)
#endif

__global__ void __launch_bounds__(UPD_THREADS)
update_validate_kernel(int64_t n_rows, int64_t n_cols, const int32_t *__restrict__ rb,
                       const int32_t *__restrict__ re, const int32_t *__restrict__ cap,
                       const int32_t *__restrict__ col, int64_t n_upd,
                       const int32_t *__restrict__ upd, const int32_t *__restrict__ dptr,
                       const int32_t *__restrict__ dcol, const int32_t *__restrict__ iptr,
                       const int32_t *__restrict__ icol, UpdWs *ws)
{
    pdl_enter();
    n_upd = *(volatile long long *)&ws->n_eff;  // <= the launch's bound (init kernel)
    const int lane = threadIdx.x & 31;
    const int64_t wid = (int64_t)blockIdx.x * (UPD_THREADS / 32) + (threadIdx.x >> 5);
    if (!ACSR_UPD_SUB) {
        if (wid < n_upd) validate_row(wid, lane, n_rows, n_cols, rb, re, cap, col, upd, dptr, dcol, iptr, icol, ws);
        return;
    }
    const int64_t ibase = wid * SUB_R;
    if (ibase >= n_upd) return;
    const int s = lane / SUB_W, li = lane % SUB_W;
    const unsigned smask = 0xFFu << (s * SUB_W);
    const int64_t i = ibase + s;
    const bool has = i < n_upd;
    int r = has ? __ldg(upd + i) : 0;
    const bool rok = has && r >= 0 && r < n_rows;
    const int b = rok ? __ldg(rb + r) : 0, e = rok ? __ldg(re + r) : 0;
    const unsigned long_any = __ballot_sync(0xffffffffu, rok && e - b > SUB_MAX);
    if (long_any) {  // a longer row in this warp: full-warp validation, row by row
        for (int q = 0; q < SUB_R; q++)
            if (ibase + q < n_upd)
                validate_row(ibase + q, lane, n_rows, n_cols, rb, re, cap, col, upd, dptr, dcol, iptr, icol, ws);
        return;
    }
    int code = ACSR_OK;
    if (has && (!rok || (i > 0 && r <= __ldg(upd + i - 1)))) code = ACSR_ERR_INVALID_VALUE;
    const int d0 = (has && dptr) ? __ldg(dptr + i) : 0, d1 = (has && dptr) ? __ldg(dptr + i + 1) : 0;
    const int i0 = has ? __ldg(iptr + i) : 0, i1 = has ? __ldg(iptr + i + 1) : 0;
    bool bad = false;
    for (int j = d0 + 1 + li; j < d1; j += SUB_W) bad |= __ldg(dcol + j) < __ldg(dcol + j - 1);
    for (int j = i0 + li; j < i1; j += SUB_W) {
        const int c = __ldg(icol + j);
        bad |= (c < 0 || c >= n_cols);
    }
    if (__ballot_sync(0xffffffffu, bad) & smask) code = code ? code : ACSR_ERR_INVALID_VALUE;
    int dels = 0;
    if (code == ACSR_OK && d1 > d0)
        for (int k = b + li; k < e; k += SUB_W) dels += member(dcol, d0, d1, __ldg(col + k)) ? 1 : 0;
#pragma unroll
    for (int o = SUB_W / 2; o > 0; o >>= 1) dels += __shfl_xor_sync(0xffffffffu, dels, o, SUB_W);
    if (code == ACSR_OK && has) {
        const long long new_len = (long long)(e - b) - dels + (i1 - i0);
        if (new_len > __ldg(cap + r)) code = ACSR_ERR_CAPACITY;
    }
    if (has && code != ACSR_OK && li == 0) atomicMin(&ws->key, ((unsigned long long)i << 3) | (unsigned)code);
}

__device__ __forceinline__ int block_exclusive_scan(int v, int &total, int *sh)
{
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int incl = v;
    for (int d = 1; d < 32; d <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += t;
    }
    if (lane == 31) sh[w] = incl;
    __syncthreads();
    if (w == 0) {
        const int x = lane < UPD_THREADS / 32 ? sh[lane] : 0;
        int xi = x;
        for (int d = 1; d < 32; d <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, xi, d);
            if (lane >= d) xi += t;
        }
        if (lane < UPD_THREADS / 32) sh[lane] = xi - x;
        if (lane == UPD_THREADS / 32 - 1) sh[32] = xi;
    }
    __syncthreads();
    const int r = sh[w] + incl - v;
    total = sh[32];
    __syncthreads();
    return r;
}

// capacity check of the long rows (one CTA per long update, grid-strided over the list)
__global__ void __launch_bounds__(UPD_THREADS)
update_validate_long_kernel(const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                            const int32_t *__restrict__ cap, const int32_t *__restrict__ col,
                            const int32_t *__restrict__ upd, const int32_t *__restrict__ dptr,
                            const int32_t *__restrict__ dcol, const int32_t *__restrict__ iptr, UpdWs *ws,
                            int del_cap)
{
    pdl_enter();
    __shared__ int sh[33];
    extern __shared__ int32_t sdel[];
    const unsigned n_long = *(volatile unsigned *)&ws->n_long;
    for (unsigned j = blockIdx.x; j < n_long; j += gridDim.x) {
        const int i = ws->long_list[j];
        const int r = __ldg(upd + i);
        const int b = __ldg(rb + r), e = __ldg(re + r);
        const int d0 = __ldg(dptr + i), d1 = __ldg(dptr + i + 1);
        const int m = d1 - d0;
        const bool use_s = m <= del_cap;
        if (use_s) {
            for (int t = threadIdx.x; t < m; t += UPD_THREADS) sdel[t] = __ldg(dcol + d0 + t);
            __syncthreads();
        }
        int dels = 0;
        for (int k = b + threadIdx.x; k < e; k += UPD_THREADS) {
            const int c = __ldg(col + k);
            dels += (use_s ? member_s(sdel, m, c) : member(dcol, d0, d1, c)) ? 1 : 0;
        }
        int total;
        block_exclusive_scan(dels, total, sh);
        const long long new_len = (long long)(e - b) - total + (__ldg(iptr + i + 1) - __ldg(iptr + i));
        if (threadIdx.x == 0 && new_len > __ldg(cap + r))
            atomicMin(&ws->key, ((unsigned long long)i << 3) | (unsigned)ACSR_ERR_CAPACITY);
    }
}

// stable in-place compaction + append of the long rows: chunks of 4 * UPD_THREADS entries,
// thread t owns 4 consecutive entries; every entry of a chunk is read before any write
// (a destination never passes its source), kept entries move to w + block prefix.
template <typename T>
__global__ void __launch_bounds__(UPD_THREADS)
update_apply_long_kernel(const int32_t *__restrict__ rb, int32_t *__restrict__ re, int32_t *__restrict__ col,
                         T *__restrict__ val, const int32_t *__restrict__ upd, const int32_t *__restrict__ dptr,
                         const int32_t *__restrict__ dcol, const int32_t *__restrict__ iptr,
                         const int32_t *__restrict__ icol, const T *__restrict__ ival, T one,
                         int32_t *__restrict__ outdeg, UpdWs *ws, int del_cap)
{
    pdl_enter();
    __shared__ int sh[33];
    extern __shared__ int32_t sdel[];
    if (*(volatile unsigned long long *)&ws->key != NO_FAIL) return;
    const unsigned n_long = *(volatile unsigned *)&ws->n_long;
    constexpr int E = 4;
    for (unsigned j = blockIdx.x; j < n_long; j += gridDim.x) {
        const int i = ws->long_list[j];
        const int r = __ldg(upd + i);
        const int b = __ldg(rb + r), e = re[r];
        const int d0 = __ldg(dptr + i), d1 = __ldg(dptr + i + 1);
        const int m = d1 - d0;
        const bool use_s = m <= del_cap;
        if (use_s) {
            for (int t = threadIdx.x; t < m; t += UPD_THREADS) sdel[t] = __ldg(dcol + d0 + t);
            __syncthreads();
        }
        int w = b;
        for (int k0 = b; k0 < e; k0 += E * UPD_THREADS) {
            int c[E];
            T v[E];
            bool keep[E], del[E];
            int cnt = 0;
#pragma unroll
            for (int q = 0; q < E; q++) {
                const int kk = k0 + threadIdx.x * E + q;
                const bool valid = kk < e;
                c[q] = valid ? col[kk] : 0;
                v[q] = (val && valid) ? val[kk] : T();
                del[q] = valid && (use_s ? member_s(sdel, m, c[q]) : member(dcol, d0, d1, c[q]));
                keep[q] = valid && !del[q];
                cnt += keep[q] ? 1 : 0;
            }
            int total;
            int dst = w + block_exclusive_scan(cnt, total, sh);  // includes a __syncthreads: reads done
#pragma unroll
            for (int q = 0; q < E; q++) {
                if (keep[q]) {
                    col[dst] = c[q];
                    if (val) val[dst] = v[q];
                    dst++;
                }
                if (del[q] && outdeg) atomicSub(outdeg + c[q], 1);
            }
            w += total;
            __syncthreads();
        }
        const int i0 = __ldg(iptr + i), i1 = __ldg(iptr + i + 1);
        for (int q = i0 + threadIdx.x; q < i1; q += UPD_THREADS) {
            const int cc = __ldg(icol + q);
            col[w + (q - i0)] = cc;
            if (val) val[w + (q - i0)] = ival ? ival[q] : one;
            if (outdeg) atomicAdd(outdeg + cc, 1);
        }
        if (threadIdx.x == 0) re[r] = w + (i1 - i0);
        __syncthreads();
    }
}

// compaction + append of update i by one full warp (called warp-uniformly)
template <typename T>
__device__ __forceinline__ void apply_row(int64_t i, int lane, const int32_t *__restrict__ rb,
                                          int32_t *__restrict__ re, int32_t *__restrict__ col,
                                          T *__restrict__ val, const int32_t *__restrict__ upd,
                                          const int32_t *__restrict__ dptr, const int32_t *__restrict__ dcol,
                                          const int32_t *__restrict__ iptr, const int32_t *__restrict__ icol,
                                          const T *__restrict__ ival, T one, int32_t *__restrict__ outdeg)
{
    const unsigned lt = (1u << lane) - 1u;
    const int r = __ldg(upd + i);
    const int d0 = dptr ? __ldg(dptr + i) : 0, d1 = dptr ? __ldg(dptr + i + 1) : 0;
    const int i0 = __ldg(iptr + i), i1 = __ldg(iptr + i + 1);  // (independent loads first)
    const int b = __ldg(rb + r), e = re[r];
    int w = e;
    if (d1 > d0 && e - b > LONG_ROW) return;  // update_apply_long_kernel
    if (d1 > d0) {
        w = b;
        const int m = d1 - d0;
        const bool wr = ACSR_UPD_WARPREG && m <= 32;
        const int dreg = (wr && lane < m) ? __ldg(dcol + d0 + lane) : 0;
        for (int k0 = b; k0 < e; k0 += 32) {
            int kk = k0 + lane;
            bool valid = kk < e;
            int c = valid ? col[kk] : 0;
            T v = T();
            if (val && valid) v = val[kk];
            const bool hw = wr ? member_w(dreg, m, c) : false;  // every lane shuffles (wr is warp-uniform)
            bool del = valid && (wr ? hw : member(dcol, d0, d1, c));
            bool keep = valid && !del;
            unsigned m = __ballot_sync(0xffffffffu, keep);
            __syncwarp();  // every lane has read its source before anyone writes
            if (keep) {
                int dst = w + __popc(m & lt);
                col[dst] = c;
                if (val) val[dst] = v;
            }
            if (del && outdeg) atomicSub(outdeg + c, 1);
            w += __popc(m);
            __syncwarp();
        }
    }
    for (int j = i0 + lane; j < i1; j += 32) {
        int c = __ldg(icol + j);
        col[w + (j - i0)] = c;
        if (val) val[w + (j - i0)] = ival ? ival[j] : one;
        if (outdeg) atomicAdd(outdeg + c, 1);
    }
    if (lane == 0) re[r] = w + (i1 - i0);
}

template <typename T>
__global__ void __launch_bounds__(UPD_THREADS)
update_apply_kernel(const int32_t *__restrict__ rb, int32_t *__restrict__ re,
                    int32_t *__restrict__ col, T *__restrict__ val, int64_t n_upd,
                    const int32_t *__restrict__ upd, const int32_t *__restrict__ dptr,
                    const int32_t *__restrict__ dcol, const int32_t *__restrict__ iptr,
                    const int32_t *__restrict__ icol, const T *__restrict__ ival, T one,
                    int32_t *__restrict__ outdeg, const UpdWs *ws, int32_t *__restrict__ status)
{
    pdl_enter();
    const unsigned long long k = *(volatile const unsigned long long *)&ws->key;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        status[0] = k == NO_FAIL ? ACSR_OK : (int32_t)(k & 7);
        status[1] = k == NO_FAIL ? -1 : (int32_t)(k >> 3);
    }
    if (k != NO_FAIL) return;  // all-or-nothing
    n_upd = *(volatile const long long *)&ws->n_eff;
    const int lane = threadIdx.x & 31;
    const int64_t wid = (int64_t)blockIdx.x * (UPD_THREADS / 32) + (threadIdx.x >> 5);
    if (!ACSR_UPD_SUB) {
        if (wid < n_upd) apply_row<T>(wid, lane, rb, re, col, val, upd, dptr, dcol, iptr, icol, ival, one, outdeg);
        return;
    }
    const int64_t ibase = wid * SUB_R;
    if (ibase >= n_upd) return;
    const int s = lane / SUB_W, li = lane % SUB_W;
    const int64_t i = ibase + s;
    const bool has = i < n_upd;
    const int r = has ? __ldg(upd + i) : 0;
    const int b = has ? __ldg(rb + r) : 0, e = has ? re[r] : 0;
    if (__ballot_sync(0xffffffffu, has && e - b > SUB_MAX)) {  // the same decision as validation
        for (int q = 0; q < SUB_R; q++)
            if (ibase + q < n_upd)
                apply_row<T>(ibase + q, lane, rb, re, col, val, upd, dptr, dcol, iptr, icol, ival, one, outdeg);
        return;
    }
    const int d0 = (has && dptr) ? __ldg(dptr + i) : 0, d1 = (has && dptr) ? __ldg(dptr + i + 1) : 0;
    int w = e;
    if (__ballot_sync(0xffffffffu, d1 > d0)) {
        // stable in-place compaction, SUB_W entries per round; the round count is the warp's
        // maximum so the ballots are warp-uniform (rows <= SUB_MAX entries)
        const int len = d1 > d0 ? e - b : 0;
        const int lmax = __reduce_max_sync(0xffffffffu, (unsigned)len);
        if (d1 > d0) w = b;
        const unsigned lt = (1u << li) - 1u;
        for (int t0 = 0; t0 < lmax; t0 += SUB_W) {
            const bool valid = t0 + li < len;
            const int kk = b + t0 + li;
            const int c = valid ? col[kk] : 0;
            T v = T();
            if (val && valid) v = val[kk];
            const bool del = valid && member(dcol, d0, d1, c);
            const bool keep = valid && !del;
            const unsigned m = (__ballot_sync(0xffffffffu, keep) >> (s * SUB_W)) & 0xFFu;
            __syncwarp();  // every lane has read its source before anyone writes
            if (keep) {
                const int dst = w + __popc(m & lt);
                col[dst] = c;
                if (val) val[dst] = v;
            }
            if (del && outdeg) atomicSub(outdeg + c, 1);
            w += __popc(m);
            __syncwarp();
        }
    }
    if (has) {
        const int i0 = __ldg(iptr + i), i1 = __ldg(iptr + i + 1);
        for (int j = i0 + li; j < i1; j += SUB_W) {
            const int c = __ldg(icol + j);
            col[w + (j - i0)] = c;
            if (val) val[w + (j - i0)] = ival ? ival[j] : one;
            if (outdeg) atomicAdd(outdeg + c, 1);
        }
        if (li == 0) re[r] = w + (i1 - i0);
    }
}

// re-layout: copy row r from [ob[r], oe[r]) to [nb[r], nb[r] + len) (warp per row)
template <typename T>
__global__ void __launch_bounds__(UPD_THREADS)
relayout_kernel(int64_t n_rows, const int32_t *__restrict__ ob, const int32_t *__restrict__ oe,
                const int32_t *__restrict__ ocol, const T *__restrict__ oval,
                const int32_t *__restrict__ nb, int32_t *__restrict__ ne, int32_t *__restrict__ ncol,
                T *__restrict__ nval)
{
    const int lane = threadIdx.x & 31;
    const int64_t r = (int64_t)blockIdx.x * (UPD_THREADS / 32) + (threadIdx.x >> 5);
    if (r >= n_rows) return;
    const int b = __ldg(ob + r), e = __ldg(oe + r), d = __ldg(nb + r);
    for (int k = lane; k < e - b; k += 32) {
        ncol[d + k] = __ldg(ocol + b + k);
        if (oval) nval[d + k] = __ldg(oval + b + k);
    }
    if (lane == 0) ne[r] = d + (e - b);
}

}  // namespace acsr

using namespace acsr;

extern "C" acsr_status acsr_relayout(acsr_dtype dt, int64_t n_rows, const int32_t *old_begin,
                                     const int32_t *old_end, const int32_t *old_col,
                                     const void *old_val, const int32_t *new_begin, int32_t *new_end,
                                     int32_t *new_col, void *new_val, cudaStream_t stream)
{
    if (n_rows < 0 || (dt != ACSR_F32 && dt != ACSR_F64) ||
        (n_rows > 0 && (!old_begin || !old_end || !new_begin || !new_end)) ||
        ((old_val == nullptr) != (new_val == nullptr))) {
        acsr_set_error("acsr_relayout: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (n_rows == 0) return ACSR_OK;
    const int wpb = UPD_THREADS / 32;
    const int64_t blocks = (n_rows + wpb - 1) / wpb;
    if (dt == ACSR_F64)
        relayout_kernel<uint64_t><<<(unsigned)blocks, UPD_THREADS, 0, stream>>>(
            n_rows, old_begin, old_end, old_col, (const uint64_t *)old_val, new_begin, new_end, new_col,
            (uint64_t *)new_val);
    else
        relayout_kernel<uint32_t><<<(unsigned)blocks, UPD_THREADS, 0, stream>>>(
            n_rows, old_begin, old_end, old_col, (const uint32_t *)old_val, new_begin, new_end, new_col,
            (uint32_t *)new_val);
    return acsr_check_launch("acsr_relayout");
}

extern "C" size_t acsr_update_workspace_bytes(int64_t n_upd)
{
    return align_up(offsetof(UpdWs, long_list) + sizeof(int32_t) * (size_t)(n_upd > 0 ? n_upd : 1), 256);
}

__global__ void update_init_kernel(UpdWs *ws, int64_t n_host, const int64_t *n_dev)
{
    pdl_enter();
    ws->key = NO_FAIL;
    ws->n_long = 0;
    long long n = n_host;
    if (n_dev) {  // acsr_update_edges_dev: the batch size lives on the device
        n = *n_dev;
        if (n < 0 || n > n_host) {  // outside the launch's bound: the batch is rejected whole
            ws->key = (unsigned long long)ACSR_ERR_INVALID_VALUE;  // index 0
            n = 0;
        }
    }
    ws->n_eff = n;
}

static acsr_status update_impl(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                         const int32_t *row_begin, int32_t *row_end,
                                         const int32_t *row_cap, int32_t *col_idx, void *values,
                                         int64_t n_upd, const int32_t *upd_rows,
                                         const int32_t *del_ptr, const int32_t *del_cols,
                                         const int32_t *ins_ptr, const int32_t *ins_cols,
                                         const void *ins_vals, int32_t *outdeg, int32_t *status,
                                         void *ws, size_t ws_bytes, cudaStream_t stream, const int64_t *n_dev)
{
    if (n_rows < 0 || n_cols < 0 || n_upd < 0 || !status || (dt != ACSR_F32 && dt != ACSR_F64) ||
        (n_upd > 0 && (!row_begin || !row_end || !row_cap || !col_idx || !upd_rows || !ins_ptr)) ||
        ((del_ptr == nullptr) != (del_cols == nullptr) && del_ptr != nullptr && n_upd > 0)) {
        acsr_set_error("acsr_update_edges: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!ws || ws_bytes < acsr_update_workspace_bytes(n_upd)) {
        acsr_set_error("acsr_update_edges: workspace too small");
        return ACSR_ERR_WORKSPACE;
    }
    UpdWs *uw = (UpdWs *)ws;
    launch_pdl(update_init_kernel, 1, 1, 0, stream, uw, n_upd, n_dev);
    const int long_grid = 4 * acsr_num_sms();
    // hub-row delete lists in shared memory (ACSR_UPD_SMEM=0: global binary search, A/B)
    static int del_cap = -1;
    if (del_cap < 0) {
        const char *e = getenv("ACSR_UPD_SMEM");
        del_cap = (e && e[0] == '0') ? 0 : DEL_SMEM_MAX;
        if (del_cap) {
            const int bytes = (int)(sizeof(int32_t) * DEL_SMEM_MAX);
            if (cudaFuncSetAttribute(update_validate_long_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess ||
                cudaFuncSetAttribute(update_apply_long_kernel<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess ||
                cudaFuncSetAttribute(update_apply_long_kernel<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess) {
                cudaGetLastError();
                del_cap = 0;
            }
        }
    }
    const size_t long_smem = sizeof(int32_t) * (size_t)del_cap;
    const int lgrid = del_cap ? acsr_num_sms() : long_grid;  // one 192 KB CTA per SM
    const int wpb = UPD_THREADS / 32;
    const int64_t upw = ACSR_UPD_SUB ? SUB_R : 1;  // updates per warp
    const int64_t blocks64 = n_upd > 0 ? (n_upd + wpb * upw - 1) / (wpb * upw) : 1;
    if (blocks64 > 0x7fffffff) return ACSR_ERR_INVALID_VALUE;
    const int blocks = (int)blocks64;
    if (n_upd > 0)
        launch_pdl(update_validate_kernel, blocks, UPD_THREADS, 0, stream, n_rows, n_cols, row_begin, row_end,
                                                                   row_cap, col_idx, n_upd, upd_rows,
                                                                   del_ptr, del_cols, ins_ptr, ins_cols,
                                                                   uw);
    if (n_upd > 0 && del_ptr)
        launch_pdl(update_validate_long_kernel, lgrid, UPD_THREADS, long_smem, stream, row_begin, row_end, row_cap,
                   col_idx, upd_rows, del_ptr, del_cols, ins_ptr, uw, del_cap);
    if (dt == ACSR_F64) {
        uint64_t one;
        double d1 = 1.0;
        memcpy(&one, &d1, 8);
        launch_pdl(update_apply_kernel<uint64_t>, blocks, UPD_THREADS, 0, stream, 
            row_begin, row_end, col_idx, (uint64_t *)values, n_upd, upd_rows, del_ptr, del_cols, ins_ptr,
            ins_cols, (const uint64_t *)ins_vals, one, outdeg, uw, status);
        if (n_upd > 0 && del_ptr)
            launch_pdl(update_apply_long_kernel<uint64_t>, lgrid, UPD_THREADS, long_smem, stream,
                row_begin, row_end, col_idx, (uint64_t *)values, upd_rows, del_ptr, del_cols, ins_ptr, ins_cols,
                (const uint64_t *)ins_vals, one, outdeg, uw, del_cap);
    } else {
        uint32_t one;
        float f1 = 1.0f;
        memcpy(&one, &f1, 4);
        launch_pdl(update_apply_kernel<uint32_t>, blocks, UPD_THREADS, 0, stream, 
            row_begin, row_end, col_idx, (uint32_t *)values, n_upd, upd_rows, del_ptr, del_cols, ins_ptr,
            ins_cols, (const uint32_t *)ins_vals, one, outdeg, uw, status);
        if (n_upd > 0 && del_ptr)
            launch_pdl(update_apply_long_kernel<uint32_t>, lgrid, UPD_THREADS, long_smem, stream,
                row_begin, row_end, col_idx, (uint32_t *)values, upd_rows, del_ptr, del_cols, ins_ptr, ins_cols,
                (const uint32_t *)ins_vals, one, outdeg, uw, del_cap);
    }
    return acsr_check_launch("acsr_update_edges");
}

extern "C" acsr_status acsr_update_edges(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                         const int32_t *row_begin, int32_t *row_end,
                                         const int32_t *row_cap, int32_t *col_idx, void *values,
                                         int64_t n_upd, const int32_t *upd_rows,
                                         const int32_t *del_ptr, const int32_t *del_cols,
                                         const int32_t *ins_ptr, const int32_t *ins_cols,
                                         const void *ins_vals, int32_t *outdeg, int32_t *status,
                                         void *ws, size_t ws_bytes, cudaStream_t stream)
{
    return update_impl(dt, n_rows, n_cols, row_begin, row_end, row_cap, col_idx, values, n_upd, upd_rows, del_ptr,
                       del_cols, ins_ptr, ins_cols, ins_vals, outdeg, status, ws, ws_bytes, stream, nullptr);
}

extern "C" acsr_status acsr_update_edges_dev(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                             const int32_t *row_begin, int32_t *row_end,
                                             const int32_t *row_cap, int32_t *col_idx, void *values,
                                             int64_t n_upd_max, const int64_t *n_upd_dev,
                                             const int32_t *upd_rows, const int32_t *del_ptr,
                                             const int32_t *del_cols, const int32_t *ins_ptr,
                                             const int32_t *ins_cols, const void *ins_vals, int32_t *outdeg,
                                             int32_t *status, void *ws, size_t ws_bytes, cudaStream_t stream)
{
    if (!n_upd_dev) {
        acsr_set_error("acsr_update_edges_dev: n_upd_dev is required");
        return ACSR_ERR_INVALID_VALUE;
    }
    return update_impl(dt, n_rows, n_cols, row_begin, row_end, row_cap, col_idx, values, n_upd_max, upd_rows,
                       del_ptr, del_cols, ins_ptr, ins_cols, ins_vals, outdeg, status, ws, ws_bytes, stream,
                       n_upd_dev);
}
