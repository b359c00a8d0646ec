// acsr_comm.cu -- the multi-GPU exchange owned by the library (§VIII row split,
// reading Q19).
//
// Row-partitioned PageRank needs, after every step, (1) every rank's slice of the scaled
// vector xs' = PR'/outdeg in every rank's replicated xs and (2) the global Delta^2 of the
// convergence test (Alg. 5; reading Q9).  Both run here on the caller's stream,
// right behind the fused step kernel, over NCCL (NVLink / NVSwitch inside a node):
//   * one in-place ncclAllGather of the equal-length (padded) slices, and
//   * one ncclAllGather of the ranks' EXACT 192-bit fixed-point Delta^2 partials, which a
//     one-warp kernel then adds in rank order: the global Delta^2 -- and with it the
//     device-side stop decision -- is the same bits on every rank and equal to the
//     single-GPU value (fixed-point sums do not depend on the order or the partition).
// Also here: acsr_partition (O8's nnz-balanced contiguous split, computed on the device
// with a CUB prefix sum + binary search) and a byte all-gather for setup-time layout work.
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdlib.h>
#include <string.h>

#include <cub/device/device_scan.cuh>
#include <thrust/iterator/counting_iterator.h>
#include <thrust/iterator/transform_iterator.h>

#include "acsr_internal.cuh"

struct acsr_comm {
    ncclComm_t nccl = nullptr;
    int nranks = 0, rank = 0, device = 0;
    uint64_t *d2 = nullptr;  // device [(nranks + 1) * 3]: own partial, then every rank's
};

static acsr_status nccl_fail(const char *what, ncclResult_t r)
{
    acsr_set_error("%s: %s", what, ncclGetErrorString(r));
    return ACSR_ERR_NCCL;
}

namespace acsr {

// global Delta^2 = exact sum of the gathered partials (rank order; the sum is exact, so
// any order gives the same bits); the device-side stop flag for every rank alike
__global__ void comm_d2_finalize_kernel(const uint64_t *__restrict__ parts, int nranks, double *delta2,
                                        int32_t *ctrl, double eps2)
{
    if (threadIdx.x != 0) return;
    if (ctrl && *(volatile int32_t *)ctrl) return;  // converged (or plan error) earlier: step was a no-op
    uint64_t hi = 0, mid = 0, lo = 0;
    for (int q = 0; q < nranks; q++) fix192_merge(hi, mid, lo, parts[3 * q], parts[3 * q + 1], parts[3 * q + 2]);
    const double d2 = fix192_to_double(hi, mid, lo);
    *delta2 = d2;
    if (ctrl && d2 <= eps2) ctrl[0] = 1;
}

__global__ void split_search_kernel(const int64_t *__restrict__ incl, int64_t n, int P, int64_t align,
                                    int64_t *splits)
{
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k > P) return;
    if (k == 0 || k == P || n == 0) {
        splits[k] = (k == P) ? n : 0;
        return;
    }
    const int64_t total = incl[n - 1];
    const int64_t target = ((int64_t)k * total + P - 1) / P;  // ceil(k * total / P)
    // min r in [0, n] with sum_{r' < r} cost(r') = (r ? incl[r-1] : 0) >= target
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        const int64_t mid = (lo + hi) / 2;
        const int64_t f = mid ? incl[mid - 1] : 0;
        if (f >= target) hi = mid;
        else lo = mid + 1;
    }
    if (align > 1) {  // reading R7: every rank starts on an aligned row
        lo = (lo + align - 1) / align * align;
        if (lo > n) lo = n;
    }
    splits[k] = lo;
}

struct RowCost {
    const int32_t *rb, *re;
    int64_t b_nnz, b_row;
    __host__ __device__ int64_t operator()(int64_t r) const
    {
        const int64_t len = (int64_t)(re ? re[r] : rb[r + 1]) - rb[r];
        return b_nnz * len + b_row;
    }
};

}  // namespace acsr

using namespace acsr;

extern "C" acsr_status acsr_comm_get_unique_id(void *id)
{
    if (!id) {
        acsr_set_error("acsr_comm_get_unique_id: id is NULL");
        return ACSR_ERR_INVALID_VALUE;
    }
    ncclUniqueId u;
    const ncclResult_t r = ncclGetUniqueId(&u);
    if (r != ncclSuccess) return nccl_fail("acsr_comm_get_unique_id", r);
    memcpy(id, u.internal, NCCL_UNIQUE_ID_BYTES);
    return ACSR_OK;
}

extern "C" acsr_status acsr_comm_init(acsr_comm **out, int nranks, int rank, const void *id)
{
    static_assert(ACSR_COMM_ID_BYTES == NCCL_UNIQUE_ID_BYTES, "unique id size");
    if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks) {
        acsr_set_error("acsr_comm_init: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    *out = nullptr;
    acsr_comm *c = new acsr_comm();
    c->nranks = nranks;
    c->rank = rank;
    cudaGetDevice(&c->device);
    cudaError_t e = cudaMalloc(&c->d2, sizeof(uint64_t) * 3 * (size_t)(nranks + 1));
    if (e != cudaSuccess) {
        acsr_set_error("acsr_comm_init: %s", cudaGetErrorString(e));
        delete c;
        return ACSR_ERR_CUDA;
    }
    cudaMemset(c->d2, 0, sizeof(uint64_t) * 3 * (size_t)(nranks + 1));
    ncclUniqueId u;
    memcpy(u.internal, id, NCCL_UNIQUE_ID_BYTES);
    const ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, u, rank);
    if (r != ncclSuccess) {
        cudaFree(c->d2);
        delete c;
        return nccl_fail("acsr_comm_init (ncclCommInitRank)", r);
    }
    *out = c;
    return ACSR_OK;
}

extern "C" acsr_status acsr_comm_destroy(acsr_comm *c)
{
    if (!c) return ACSR_OK;
    acsr_status st = ACSR_OK;
    if (c->nccl) {
        const ncclResult_t r = ncclCommDestroy(c->nccl);
        if (r != ncclSuccess) st = nccl_fail("acsr_comm_destroy", r);
    }
    cudaFree(c->d2);
    delete c;
    return st;
}

extern "C" acsr_status acsr_comm_query(const acsr_comm *c, int *nranks, int *rank)
{
    if (!c) {
        acsr_set_error("acsr_comm_query: comm is NULL");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (nranks) *nranks = c->nranks;
    if (rank) *rank = c->rank;
    return ACSR_OK;
}

extern "C" acsr_status acsr_comm_allgather(acsr_comm *c, const void *send, void *recv, size_t bytes_per_rank,
                                           cudaStream_t stream)
{
    if (!c || (bytes_per_rank > 0 && (!send || !recv))) {
        acsr_set_error("acsr_comm_allgather: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (bytes_per_rank == 0) return ACSR_OK;
    const ncclResult_t r = ncclAllGather(send, recv, bytes_per_rank, ncclUint8, c->nccl, stream);
    if (r != ncclSuccess) return nccl_fail("acsr_comm_allgather", r);
    return acsr_check_launch("acsr_comm_allgather");
}

extern "C" acsr_status acsr_comm_allgatherv(acsr_comm *c, const void *send, void *recv, size_t stride_bytes,
                                            const int64_t *counts_bytes, cudaStream_t stream)
{
    if (!c || !counts_bytes || (stride_bytes > 0 && !recv)) {
        acsr_set_error("acsr_comm_allgatherv: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    for (int q = 0; q < c->nranks; q++)
        if (counts_bytes[q] < 0 || (size_t)counts_bytes[q] > stride_bytes || (q == c->rank && counts_bytes[q] && !send)) {
            acsr_set_error("acsr_comm_allgatherv: counts must lie in [0, stride_bytes]");
            return ACSR_ERR_INVALID_VALUE;
        }
    ncclResult_t r = ncclGroupStart();
    for (int q = 0; q < c->nranks && r == ncclSuccess; q++) {
        char *dst = (char *)recv + (size_t)q * stride_bytes;
        if (counts_bytes[q] > 0)
            r = ncclBroadcast(q == c->rank ? send : (const void *)dst, dst, (size_t)counts_bytes[q], ncclUint8, q, c->nccl,
                              stream);
    }
    const ncclResult_t r2 = ncclGroupEnd();
    if (r != ncclSuccess) return nccl_fail("acsr_comm_allgatherv", r);
    if (r2 != ncclSuccess) return nccl_fail("acsr_comm_allgatherv", r2);
    return acsr_check_launch("acsr_comm_allgatherv");
}

// Called by acsr_pagerank_step after the fused step kernel (which wrote its Delta^2
// partial to comm->d2[0..3)) when args->comm != NULL.
uint64_t *acsr_comm_d2_slot(acsr_comm *c) { return c->d2; }
int acsr_comm_nranks(const acsr_comm *c) { return c->nranks; }

// the xs slices: one all-gather of equal slices, or (slice_counts) one broadcast per rank
static ncclResult_t xs_exchange(const acsr_pr_args *p, acsr_comm *c, cudaStream_t stream)
{
    if (p->slice_len <= 0) return ncclSuccess;
    if (!p->slice_counts)
        return ncclAllGather(p->xs_next, p->xs_all, (size_t)p->slice_len, ncclFloat64, c->nccl, stream);
    ncclResult_t r = ncclSuccess;
    for (int q = 0; q < c->nranks && r == ncclSuccess; q++) {
        double *dst = p->xs_all + (int64_t)q * p->slice_len;
        const int64_t cnt = p->slice_counts[q];
        if (cnt > 0) r = ncclBroadcast(q == c->rank ? (const void *)p->xs_next : dst, dst, (size_t)cnt, ncclFloat64, q,
                                       c->nccl, stream);
    }
    return r;
}

static bool counts_ok(const acsr_pr_args *p)
{
    if (!p->slice_counts) return true;
    for (int q = 0; q < acsr_comm_nranks(p->comm); q++)
        if (p->slice_counts[q] < 0 || p->slice_counts[q] > p->slice_len) return false;
    return true;
}

acsr_status acsr_comm_step_exchange(const acsr_pr_args *p, cudaStream_t stream)
{
    acsr_comm *c = p->comm;
    ncclResult_t r = ncclGroupStart();
    if (r == ncclSuccess) r = xs_exchange(p, c, stream);
    if (r == ncclSuccess) r = ncclAllGather(c->d2, c->d2 + 3, 3, ncclUint64, c->nccl, stream);
    const ncclResult_t r2 = ncclGroupEnd();
    if (r != ncclSuccess) return nccl_fail("acsr_pagerank_step (exchange)", r);
    if (r2 != ncclSuccess) return nccl_fail("acsr_pagerank_step (exchange)", r2);
    comm_d2_finalize_kernel<<<1, 32, 0, stream>>>(c->d2 + 3, c->nranks, p->delta2, p->ctrl, p->eps2);
    return acsr_check_launch("acsr_pagerank_step (Delta^2 finalize)");
}


extern "C" acsr_status acsr_pagerank_init(const acsr_pr_args *p, cudaStream_t stream)
{
    if (!p || p->n_rows < 0 || (p->n_rows > 0 && (!p->x || !p->outdeg || !p->xs_next))) {
        acsr_set_error("acsr_pagerank_init: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (p->comm && (!p->xs_all || p->slice_len < 0 ||
                    p->n_cols < (int64_t)acsr_comm_nranks(p->comm) * p->slice_len)) {
        acsr_set_error("acsr_pagerank_init: with comm, xs_all [n_cols >= nranks * slice_len] is required");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (p->comm && !counts_ok(p)) {
        acsr_set_error("acsr_pagerank_init: slice_counts[q] must lie in [0, slice_len]");
        return ACSR_ERR_INVALID_VALUE;
    }
    acsr_status st = acsr_pagerank_scale(p->n_rows, p->x, p->outdeg, p->xs_next, stream);
    if (st != ACSR_OK || !p->comm) return st;
    if (p->slice_len == 0) return ACSR_OK;
    ncclResult_t r = ncclGroupStart();
    if (r == ncclSuccess) r = xs_exchange(p, p->comm, stream);
    const ncclResult_t r2 = ncclGroupEnd();
    if (r != ncclSuccess) return nccl_fail("acsr_pagerank_init (exchange)", r);
    if (r2 != ncclSuccess) return nccl_fail("acsr_pagerank_init (exchange)", r2);
    return acsr_check_launch("acsr_pagerank_init");
}

extern "C" size_t acsr_partition_workspace_bytes(int64_t n_rows)
{
    size_t temp = 0;
    auto it = thrust::make_transform_iterator(thrust::counting_iterator<int64_t>(0), RowCost{nullptr, nullptr, 0, 0});
    cub::DeviceScan::InclusiveSum(nullptr, temp, it, (int64_t *)nullptr, n_rows > 0 ? n_rows : 1);
    return align_up(sizeof(int64_t) * (size_t)(n_rows > 0 ? n_rows : 1), 256) + align_up(temp, 256);
}

extern "C" acsr_status acsr_partition(int64_t n_rows, const int32_t *row_begin, const int32_t *row_end,
                                      int64_t b_nnz, int64_t b_row, int nranks, int64_t align, int64_t *splits,
                                      void *ws, size_t ws_bytes, cudaStream_t stream)
{
    if (n_rows < 0 || nranks < 1 || !splits || b_nnz < 0 || b_row < 0 || (n_rows > 0 && !row_begin)) {
        acsr_set_error("acsr_partition: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!ws || ws_bytes < acsr_partition_workspace_bytes(n_rows)) {
        acsr_set_error("acsr_partition: workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    int64_t *incl = (int64_t *)ws;
    if (n_rows > 0) {
        char *temp = (char *)ws + align_up(sizeof(int64_t) * (size_t)n_rows, 256);
        size_t temp_bytes = ws_bytes - align_up(sizeof(int64_t) * (size_t)n_rows, 256);
        auto it = thrust::make_transform_iterator(thrust::counting_iterator<int64_t>(0),
                                                  RowCost{row_begin, row_end, b_nnz, b_row});
        const cudaError_t e = cub::DeviceScan::InclusiveSum(temp, temp_bytes, it, incl, n_rows, stream);
        if (e != cudaSuccess) {
            acsr_set_error("acsr_partition (scan): %s", cudaGetErrorString(e));
            return ACSR_ERR_CUDA;
        }
    }
    split_search_kernel<<<(nranks + 1 + 127) / 128, 128, 0, stream>>>(incl, n_rows, nranks, align, splits);
    return acsr_check_launch("acsr_partition");
}

// ---------------------------------------------------------------------------------------
// Compact (dangling-free) exchange layout of the row-partitioned PageRank (SURVEY §8(e)
// lever 2): xs_u = 0 exactly when outdeg_u = 0 (Alg. 5 with reading Q11), so only
// non-dangling vertices get a slot in the replicated xs.
namespace acsr {
__global__ void nd_to_int_kernel(int64_t n, const uint8_t *__restrict__ nd, int32_t *__restrict__ v)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
        v[i] = i < n ? (nd[i] != 0) : 0;
}

// one thread per rank: non-dangling count; Lx = max(1, max count)
__global__ void layout_counts_kernel(const int64_t *__restrict__ splits, int P, const int32_t *__restrict__ excl,
                                     int64_t *__restrict__ counts, int64_t *lx)
{
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    int64_t m = 1;
    for (int k = 0; k < P; k++) {
        const int64_t c = (int64_t)excl[splits[k + 1]] - excl[splits[k]];
        counts[k] = c;
        m = c > m ? c : m;
    }
    *lx = m;
}

__global__ void layout_pos_kernel(int64_t n, const int64_t *__restrict__ splits, int P, const uint8_t *__restrict__ nd,
                                  const int32_t *__restrict__ excl, const int64_t *__restrict__ lx,
                                  int32_t *__restrict__ pos, int rank, int32_t *__restrict__ order)
{
    const int64_t Lx = *lx;
    const int64_t lo = splits[rank], hi = splits[rank + 1];
    const int64_t nloc_nd = (int64_t)excl[hi] - excl[lo];
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int owner = 0;
        while (owner + 1 < P && splits[owner + 1] <= v) owner++;
        const bool isnd = nd[v] != 0;
        const int64_t rk = (int64_t)excl[v] - excl[splits[owner]];
        pos[v] = (int32_t)(isnd ? owner * Lx + rk : (int64_t)P * Lx);
        if (order && v >= lo && v < hi) {  // this rank's rows: non-dangling first, each group in row order
            const int64_t r = v - lo;
            const int64_t dst = isnd ? rk : nloc_nd + (r - rk);
            order[dst] = (int32_t)r;
        }
    }
}
}  // namespace acsr

extern "C" size_t acsr_exchange_layout_workspace_bytes(int64_t n_global)
{
    const size_t nn = (size_t)(n_global > 0 ? n_global : 0) + 1;
    size_t temp = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, temp, (const int32_t *)nullptr, (int32_t *)nullptr, (int)nn);
    return 2 * align_up(4 * nn, 256) + align_up(temp, 256);
}

extern "C" acsr_status acsr_exchange_layout(int64_t n_global, int nranks, const int64_t *splits, const uint8_t *nd,
                                            int rank, int32_t *pos, int32_t *order, int64_t *counts, int64_t *lx,
                                            void *ws, size_t ws_bytes, cudaStream_t stream)
{
    if (n_global < 0 || n_global >= ((int64_t)1 << 31) || nranks < 1 || rank < -1 || rank >= nranks || !splits ||
        !counts || !lx || (n_global > 0 && (!nd || !pos)) || (order && rank < 0)) {
        acsr_set_error("acsr_exchange_layout: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!ws || ws_bytes < acsr_exchange_layout_workspace_bytes(n_global)) {
        acsr_set_error("acsr_exchange_layout: workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    const size_t nn = (size_t)n_global + 1;
    int32_t *v = (int32_t *)ws;
    int32_t *excl = (int32_t *)((char *)ws + align_up(4 * nn, 256));
    void *temp = (char *)ws + 2 * align_up(4 * nn, 256);
    size_t tb = ws_bytes - 2 * align_up(4 * nn, 256);
    const int sms = acsr_num_sms();
    const int grid = (int)((int64_t)(nn + 255) / 256 < (int64_t)sms * 8 ? (int64_t)(nn + 255) / 256 : (int64_t)sms * 8);
    nd_to_int_kernel<<<grid, 256, 0, stream>>>(n_global, nd, v);
    const cudaError_t e = cub::DeviceScan::ExclusiveSum(temp, tb, v, excl, (int)nn, stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_exchange_layout (scan): %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    layout_counts_kernel<<<1, 32, 0, stream>>>(splits, nranks, excl, counts, lx);
    if (n_global > 0)
        layout_pos_kernel<<<grid, 256, 0, stream>>>(n_global, splits, nranks, nd, excl, lx, pos, rank < 0 ? 0 : rank,
                                                    order);
    return acsr_check_launch("acsr_exchange_layout");
}
