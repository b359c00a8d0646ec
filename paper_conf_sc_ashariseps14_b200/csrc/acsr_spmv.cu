// acsr_spmv.cu -- bin-specific SpMV (Alg. 2) in ONE launch, plus the
// fused PageRank step (Alg. 5).
//
// Work is cut by acsr_bin into warp-sized units (see acsr_internal.cuh):
//   heavy units   one HEAVY_CHUNK-nnz chunk of a row with > 1024 nnz; the last
//                 warp to finish a row (threadfence + atomic ticket) sums the
//                 chunk partials in chunk order (replaces the dynamic-parallelism
//                 parent/child kernels, Alg. 3/4).
//   light units   up to unit_rows(b) rows of one bin b <= 10 inside one 4096-row
//                 tile; bins 1..6 use a sub-warp of 2^{b-1} lanes per row and a
//                 width-2^{b-1} shuffle reduction (exactly Alg. 2 with reading Q6);
//                 bins 7..10 use a full warp per row; bin 0 writes +0.0 (Q2).
// Units are listed heavy-first, then tile by tile in row order; warps take units
// round-robin, so at any moment the GPU works on a narrow window of the row space
// and the CSR sectors shared by neighbouring rows of different bins are re-used
// from L2 instead of being fetched twice.
//
// Every row is summed in an order that depends only on its length and address:
// results are deterministic run to run.  Accumulation is in double for both
// ACSR_F64 and ACSR_F32 (products of floats are exact in double).
#include <cuda_runtime.h>

#include "acsr_internal.cuh"

namespace acsr {

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
    double *__restrict__ warp_part;
    // PageRank epilogue
    const double *__restrict__ x_old;
    const int32_t *__restrict__ outdeg;
    double *__restrict__ x_new;
    double *__restrict__ xs_next;
    double damping, teleport;
    double *delta2;
};

template <typename V, bool HAS_VAL, bool HAS_END, bool PR>
struct Kern {
    using A = SpmvArgs<V>;

    static __device__ __forceinline__ void row_bounds(const A &a, int r, int &beg, int &end)
    {
        beg = __ldg(a.rb + r);
        end = HAS_END ? __ldg(a.re + r) : __ldg(a.rb + r + 1);
    }

    static __device__ __forceinline__ double prod(const A &a, int k)
    {
        int c = __ldcs(a.col + k);
        double xv = (double)__ldg(a.x + c);
        if (HAS_VAL) return (double)__ldcs(a.val + k) * xv;
        return xv;
    }

    static __device__ __forceinline__ double fmac(const A &a, int k, double acc)
    {
        int c = __ldcs(a.col + k);
        double xv = (double)__ldg(a.x + c);
        if (HAS_VAL) return fma((double)__ldcs(a.val + k), xv, acc);
        return acc + xv;
    }

    // write the row result (or the PageRank epilogue for local row r)
    static __device__ __forceinline__ void finish(const A &a, int r, double s, double &d2)
    {
        if (PR) {
            double xn = a.teleport + a.damping * s;
            a.x_new[r] = xn;
            int od = __ldg(a.outdeg + r);
            a.xs_next[r] = od > 0 ? xn / (double)od : 0.0;
            double diff = xn - __ldg(a.x_old + r);
            d2 += diff * diff;
        } else {
            a.y[r] = (V)s;
        }
    }

    // bins 1..6: W = 2^{b-1} lanes per row, each lane <= 2 elements (Alg. 2)
    template <int W>
    static __device__ __forceinline__ void light_sub(const A &a, int start, int cnt, int lane, double &d2)
    {
        constexpr int RPP = 32 / W;  // rows per pass
        constexpr int U = (W >= 16) ? 2 : 4;  // passes in flight
        const int sub = lane / W, li = lane % W;
        for (int i0 = 0; i0 < cnt; i0 += RPP * U) {
            int r[U], beg[U], end[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                int i = i0 + u * RPP + sub;
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
                int k0 = beg[u] + li, k1 = k0 + W;
                double s = 0.0;
                if (k0 < end[u]) s = prod(a, k0);
                if (k1 < end[u]) s += prod(a, k1);
                acc[u] = s;
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

    // lane-strided dot over [kb, ke), 4 independent loads in flight per lane
    static __device__ __forceinline__ double strided_dot(const A &a, int kb, int ke, int lane)
    {
        double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
        int k = kb + lane;
        for (; k + 96 < ke; k += 128) {
            s0 = fmac(a, k, s0);
            s1 = fmac(a, k + 32, s1);
            s2 = fmac(a, k + 64, s2);
            s3 = fmac(a, k + 96, s3);
        }
        for (; k < ke; k += 32) s0 = fmac(a, k, s0);
        return (s0 + s1) + (s2 + s3);
    }

    // bins 7..10: a warp per row
    static __device__ __forceinline__ void light_warp(const A &a, int start, int cnt, int lane, double &d2)
    {
        int myr = lane < cnt ? __ldg(a.bin_rows + start + lane) : 0;
        int mb = 0, me = 0;
        if (lane < cnt) row_bounds(a, myr, mb, me);
        for (int i = 0; i < cnt; i++) {
            int r = __shfl_sync(0xffffffffu, myr, i);
            int beg = __shfl_sync(0xffffffffu, mb, i);
            int end = __shfl_sync(0xffffffffu, me, i);
            double s = warp_sum(strided_dot(a, beg, end, lane));
            if (lane == 0) finish(a, r, s, d2);
        }
    }

    static __device__ __forceinline__ void empty_rows(const A &a, int start, int cnt, int lane, double &d2)
    {
        for (int i = lane; i < cnt; i += 32) finish(a, __ldg(a.bin_rows + start + i), 0.0, d2);
    }

    // one HEAVY_CHUNK chunk of a long row; last arriver combines in chunk order
    static __device__ __forceinline__ void heavy(const A &a, int u, int r, int c, int lane, double &d2)
    {
        int beg, end;
        row_bounds(a, r, beg, end);
        int kb = beg + c * HEAVY_CHUNK;
        int ke = min(kb + HEAVY_CHUNK, end);
        double s = warp_sum(strided_dot(a, kb, ke, lane));
        int nch = heavy_chunks(end - beg);
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
};

template <typename V, bool HAS_VAL, bool HAS_END, bool PR>
__global__ void __launch_bounds__(SPMV_THREADS)
spmv_kernel(SpmvArgs<V> a)
{
    using K = Kern<V, HAS_VAL, HAS_END, PR>;
    const int lane = threadIdx.x & 31;
    const int gw = blockIdx.x * SPMV_WARPS + (threadIdx.x >> 5);
    const int nw = gridDim.x * SPMV_WARPS;
    const int n_units = a.hdr->n_units;
    {
        char *ws = (char *)a.hdr;
        a.units = (const int2 *)(ws + a.hdr->off_units);
        a.partial = (double *)(ws + a.hdr->off_partial);
        a.ticket = (int32_t *)(ws + a.hdr->off_ticket);
        a.warp_part = (double *)(ws + a.hdr->off_warp_part);
    }
    double d2 = 0.0;
    for (int u = gw; u < n_units; u += nw) {
        int2 d = __ldg(a.units + u);
        uint32_t y = (uint32_t)d.y;
        if (y & HEAVY_FLAG) {
            K::heavy(a, u, d.x, (int)(y & ~HEAVY_FLAG), lane, d2);
        } else {
            int b = (int)(y >> 24), cnt = (int)(y & 0xFFFFFF);
            switch (b) {
                case 0: K::empty_rows(a, d.x, cnt, lane, d2); break;
                case 1: K::template light_sub<1>(a, d.x, cnt, lane, d2); break;
                case 2: K::template light_sub<2>(a, d.x, cnt, lane, d2); break;
                case 3: K::template light_sub<4>(a, d.x, cnt, lane, d2); break;
                case 4: K::template light_sub<8>(a, d.x, cnt, lane, d2); break;
                case 5: K::template light_sub<16>(a, d.x, cnt, lane, d2); break;
                case 6: K::template light_sub<32>(a, d.x, cnt, lane, d2); break;
                default: K::light_warp(a, d.x, cnt, lane, d2); break;
            }
        }
    }
    if (PR) {
        // deterministic Delta^2: per-warp partial (fixed unit order per warp), then the
        // last warp sums the partials in warp order.
        d2 = K::warp_sum(d2);
        int last = 0;
        if (lane == 0) {
            a.warp_part[gw] = d2;
            __threadfence();
            last = (atomicAdd(&a.hdr->done_ticket, 1) == nw - 1);
        }
        last = __shfl_sync(0xffffffffu, last, 0);
        if (last) {
            __threadfence();
            double t = 0.0;
            for (int j = lane; j < nw; j += 32) t += __ldcg(a.warp_part + j);
            t = K::warp_sum(t);
            if (lane == 0) {
                *a.delta2 = t;
                a.hdr->done_ticket = 0;
            }
        }
    }
}

template <typename V, bool HAS_VAL, bool HAS_END, bool PR>
static int grid_for()
{
    static int g = 0;
    if (!g) {
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, spmv_kernel<V, HAS_VAL, HAS_END, PR>,
                                                      SPMV_THREADS, 0);
        if (per_sm < 1) per_sm = 1;
        int gg = per_sm * acsr_num_sms();
        if (gg * SPMV_WARPS > MAX_WARPS) gg = MAX_WARPS / SPMV_WARPS;
        g = gg;
    }
    return g;
}

template <typename V, bool HAS_VAL, bool HAS_END, bool PR>
static void launch(const SpmvArgs<V> &a, cudaStream_t s)
{
    spmv_kernel<V, HAS_VAL, HAS_END, PR><<<grid_for<V, HAS_VAL, HAS_END, PR>(), SPMV_THREADS, 0, s>>>(a);
}

template <typename V, bool PR>
static void dispatch(const SpmvArgs<V> &a, cudaStream_t s)
{
    bool hv = a.val != nullptr, he = a.re != nullptr;
    if (hv && he) launch<V, true, true, PR>(a, s);
    else if (hv) launch<V, true, false, PR>(a, s);
    else if (he) launch<V, false, true, PR>(a, s);
    else launch<V, false, false, PR>(a, s);
}

__global__ void pagerank_scale_kernel(int64_t n, const double *__restrict__ x,
                                      const int32_t *__restrict__ outdeg, double *__restrict__ xs)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        int od = outdeg[i];
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
    return plan_ws_bytes >= plan_layout(n_rows, 0).total;
}

extern "C" acsr_status acsr_spmv(acsr_dtype dt, int64_t n_rows, int64_t n_cols,
                                 const int32_t *row_begin, const int32_t *row_end,
                                 const int32_t *col_idx, const void *values, const void *x, void *y,
                                 const int32_t *bin_rows, const int32_t *bin_offsets, void *plan_ws,
                                 size_t plan_ws_bytes, cudaStream_t stream)
{
    if (n_rows < 0 || n_cols < 0 || n_rows >= ((int64_t)1 << 31) ||
        (dt != ACSR_F32 && dt != ACSR_F64) ||
        (n_rows > 0 && (!row_begin || !y))) {
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
        a.val = (const double *)values; a.x = (const double *)x; a.y = (double *)y;
        a.bin_rows = bin_rows; a.hdr = (PlanHeader *)plan_ws;
        dispatch<double, false>(a, stream);
    } else {
        SpmvArgs<float> a{};
        a.rb = row_begin; a.re = row_end; a.col = col_idx;
        a.val = (const float *)values; a.x = (const float *)x; a.y = (float *)y;
        a.bin_rows = bin_rows; a.hdr = (PlanHeader *)plan_ws;
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
    if (p->n_rows == 0) {
        zero_delta_kernel<<<1, 1, 0, stream>>>(p->delta2);
        return acsr_check_launch("acsr_pagerank_step(empty)");
    }
    SpmvArgs<double> a{};
    a.rb = p->row_begin; a.re = p->row_end; a.col = p->col_idx;
    a.val = nullptr; a.x = p->xs; a.y = nullptr;
    a.bin_rows = p->bin_rows; a.hdr = (PlanHeader *)p->plan_ws;
    a.x_old = p->x; a.outdeg = p->outdeg; a.x_new = p->x_new; a.xs_next = p->xs_next;
    a.damping = p->damping; a.teleport = p->teleport; a.delta2 = p->delta2;
    dispatch<double, true>(a, stream);
    return acsr_check_launch("acsr_pagerank_step");
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
