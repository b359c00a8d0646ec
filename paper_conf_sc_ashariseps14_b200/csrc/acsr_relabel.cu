// acsr_relabel.cu -- degree-ordered vertex relabelling of a PageRank in-link graph, on
// the device (an application-level preprocessing option for C4, not part of ACSR itself).
//
// PageRank gathers xs[u] = x_u / outdeg_u for every in-link u -> v (Alg. 5, P:279-291,
// reading Q12).  With R-MAT's random vertex numbering the hot (high out-degree) sources
// are scattered over the whole 537 MB xs at s26, so most gathers miss L2.  Renumbering
// the vertices by decreasing out-degree (P A P^T: rows and columns alike) packs the hot
// entries of xs at the front, where they stay in L2.  The graph persists across the
// dynamic-graph epochs, so the relabel is paid once.
//
// Steps (all on the stream, no host synchronisation):
//   1. order = vertices sorted by out-degree, descending, ties by id (CUB radix sort of
//      (outdeg, id) pairs; outdeg' = the sorted keys)
//   2. perm[order[i]] = i;  len'[i] = len(order[i])
//   3. row_ptr' = exclusive prefix of len' (CUB)
//   4. rows copied in new order with their columns renumbered c -> perm[c]: a warp per
//      32 consecutive new rows walks their concatenated entries (coalesced reads of each
//      old row run, coalesced writes); rows longer than RELABEL_LONG go to a list that
//   5. a CTA per long row copies (claimed from an atomic counter).
// Column order inside a row is kept (entry j of old row u is entry j of new row perm[u]),
// unless ACSR_RELABEL_SORT_ROWS: then every new row's columns are sorted ascending (CUB
// segmented sort), so the hot -- now small -- column ids of a row sit next to each other and
// a warp's gather instruction touches fewer 128-byte lines of xs.
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>

#include "acsr_internal.cuh"

namespace acsr {

constexpr int RELABEL_LONG = 1024;
constexpr int RELABEL_THREADS = 256;

struct RelabelLayout {
    size_t off_ids = 0, off_order = 0, off_len = 0, off_long = 0, off_ctr = 0, off_cols = 0, off_temp = 0,
           temp_bytes = 0, total = 0;
};

static RelabelLayout relabel_layout(int64_t n, int64_t nnz, unsigned flags)
{
    RelabelLayout L;
    const size_t nn = (size_t)(n > 0 ? n : 1);
    const bool sort_rows = (flags & ACSR_RELABEL_SORT_ROWS) && nnz > 0;
    size_t sort_tmp = 0, scan_tmp = 0, seg_tmp = 0;
    cub::DeviceRadixSort::SortPairsDescending(nullptr, sort_tmp, (const int32_t *)nullptr, (int32_t *)nullptr,
                                              (const int32_t *)nullptr, (int32_t *)nullptr, (int)nn);
    cub::DeviceScan::ExclusiveSum(nullptr, scan_tmp, (const int32_t *)nullptr, (int32_t *)nullptr, (int)nn + 1);
    if (sort_rows)
        cub::DeviceSegmentedSort::SortKeys(nullptr, seg_tmp, (const int32_t *)nullptr, (int32_t *)nullptr, (int)nnz,
                                           (int)nn, (const int32_t *)nullptr, (const int32_t *)nullptr);
    L.temp_bytes = sort_tmp > scan_tmp ? sort_tmp : scan_tmp;
    if (seg_tmp > L.temp_bytes) L.temp_bytes = seg_tmp;
    size_t o = 0;
    L.off_ids = o;
    o = align_up(o + 4 * nn, 256);
    L.off_order = o;
    o = align_up(o + 4 * nn, 256);
    L.off_len = o;
    o = align_up(o + 4 * (nn + 1), 256);
    L.off_long = o;
    o = align_up(o + 4 * nn, 256);
    L.off_ctr = o;
    o = align_up(o + 16, 256);
    L.off_cols = o;  // unsorted relabelled columns (ACSR_RELABEL_SORT_ROWS)
    o = align_up(o + (sort_rows ? 4 * (size_t)nnz : 0), 256);
    L.off_temp = o;
    o = align_up(o + L.temp_bytes, 256);
    L.total = o;
    return L;
}

__global__ void relabel_init_kernel(int64_t n, int32_t *ids, int32_t *ctr)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        ids[i] = (int32_t)i;
    if (blockIdx.x == 0 && threadIdx.x < 4) ctr[threadIdx.x] = 0;
}

__global__ void relabel_perm_kernel(int64_t n, const int32_t *__restrict__ order, const int32_t *__restrict__ rp,
                                    int32_t *__restrict__ perm, int32_t *__restrict__ len_new)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = order[i];
        perm[u] = (int32_t)i;
        len_new[i] = rp[u + 1] - rp[u];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) len_new[n] = 0;
}

// a warp per 32 consecutive new rows: entries of the short rows concatenated, element t
// handled by lane t mod 32 (its row found by a 5-step binary search over the lanes'
// exclusive prefixes); long rows are listed for the CTA pass
__global__ void __launch_bounds__(RELABEL_THREADS)
relabel_copy_kernel(int64_t n, const int32_t *__restrict__ order, const int32_t *__restrict__ rp,
                    const int32_t *__restrict__ col, const int32_t *__restrict__ perm /* NULL: columns kept */,
                    const int32_t *__restrict__ rp_new, int32_t *__restrict__ col_new, int32_t *__restrict__ long_rows,
                    int32_t *ctr)
{
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (RELABEL_THREADS / 32);
    for (int64_t w = blockIdx.x * (int64_t)(RELABEL_THREADS / 32) + (threadIdx.x >> 5); w * 32 < n; w += warps) {
        const int64_t i = w * 32 + lane;
        int beg = 0, len = 0, dst = 0;
        if (i < n) {
            const int32_t u = order[i];
            beg = rp[u];
            len = rp[u + 1] - beg;
            dst = rp_new[i];
            if (len > RELABEL_LONG) {
                long_rows[atomicAdd(ctr, 1)] = (int32_t)i;
                len = 0;
            }
        }
        int incl = len;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += t;
        }
        const int pre = incl - len;
        const int T = __shfl_sync(0xffffffffu, incl, 31);
        for (int t0 = 0; t0 < T; t0 += 32) {
            const int t = t0 + lane;
            // row j = the last lane with pre_j <= t (rows with len 0 share their successor's
            // prefix and are skipped because the search takes the LAST such lane)
            int j = 0;
#pragma unroll
            for (int s = 16; s > 0; s >>= 1) {
                const int pj = __shfl_sync(0xffffffffu, pre, j + s);
                if (pj <= t) j += s;
            }
            const int bj = __shfl_sync(0xffffffffu, beg, j);
            const int dj = __shfl_sync(0xffffffffu, dst, j);
            const int pj = __shfl_sync(0xffffffffu, pre, j);
            if (t < T) {
                const int e = t - pj;
                const int c = __ldcs(col + bj + e);
                col_new[dj + e] = perm ? perm[c] : c;
            }
        }
    }
}

// a CTA per long row (claimed from ctr[1] over the ctr[0] listed rows)
__global__ void __launch_bounds__(1024)
relabel_long_kernel(const int32_t *__restrict__ order, const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
                    const int32_t *__restrict__ perm, const int32_t *__restrict__ rp_new, int32_t *__restrict__ col_new,
                    const int32_t *__restrict__ long_rows, int32_t *ctr)
{
    __shared__ int s_i;
    for (;;) {
        if (threadIdx.x == 0) {
            const int k = atomicAdd(ctr + 1, 1);
            s_i = k < *(volatile int32_t *)ctr ? long_rows[k] : -1;
        }
        __syncthreads();
        const int i = s_i;
        __syncthreads();
        if (i < 0) break;
        const int32_t u = order[i];
        const int beg = rp[u], len = rp[u + 1] - beg, dst = rp_new[i];
        for (int e = threadIdx.x; e < len; e += blockDim.x) {
            const int c = __ldcs(col + beg + e);
            col_new[dst + e] = perm ? perm[c] : c;
        }
    }
}

}  // namespace acsr

using namespace acsr;

extern "C" size_t acsr_relabel_workspace_bytes(int64_t n, int64_t nnz, unsigned flags)
{
    return relabel_layout(n, nnz, flags).total;
}

extern "C" acsr_status acsr_degree_relabel(int64_t n, int64_t nnz, const int32_t *row_ptr, const int32_t *col_idx,
                                           const int32_t *outdeg, int32_t *row_ptr_out, int32_t *col_out,
                                           int32_t *outdeg_out, int32_t *perm_out, unsigned flags, void *ws,
                                           size_t ws_bytes, cudaStream_t stream)
{
    if (n < 0 || n >= ((int64_t)1 << 31) - 1 || nnz < 0 || nnz >= ((int64_t)1 << 31) ||
        (flags & ~(unsigned)ACSR_RELABEL_SORT_ROWS) ||
        (n > 0 && (!row_ptr || !outdeg || !row_ptr_out || !outdeg_out || !perm_out))) {
        acsr_set_error("acsr_degree_relabel: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    const RelabelLayout L = relabel_layout(n, nnz, flags);
    const bool sort_rows = (flags & ACSR_RELABEL_SORT_ROWS) && nnz > 0 && col_idx && col_out;
    if (!ws || ws_bytes < L.total) {
        acsr_set_error("acsr_degree_relabel: workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    if (n == 0) {
        cudaMemsetAsync(row_ptr_out, 0, sizeof(int32_t), stream);
        return acsr_check_launch("acsr_degree_relabel");
    }
    char *w = (char *)ws;
    int32_t *ids = (int32_t *)(w + L.off_ids), *order = (int32_t *)(w + L.off_order);
    int32_t *len_new = (int32_t *)(w + L.off_len), *long_rows = (int32_t *)(w + L.off_long);
    int32_t *ctr = (int32_t *)(w + L.off_ctr);
    void *temp = w + L.off_temp;
    const int sms = acsr_num_sms();
    const int grid = (int)((n + RELABEL_THREADS - 1) / RELABEL_THREADS < (int64_t)sms * 8
                               ? (n + RELABEL_THREADS - 1) / RELABEL_THREADS : (int64_t)sms * 8);
    relabel_init_kernel<<<grid, RELABEL_THREADS, 0, stream>>>(n, ids, ctr);
    size_t tb = L.temp_bytes;
    cudaError_t e = cub::DeviceRadixSort::SortPairsDescending(temp, tb, outdeg, outdeg_out, ids, order, (int)n, 0,
                                                              32, stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_degree_relabel (sort): %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    relabel_perm_kernel<<<grid, RELABEL_THREADS, 0, stream>>>(n, order, row_ptr, perm_out, len_new);
    tb = L.temp_bytes;
    e = cub::DeviceScan::ExclusiveSum(temp, tb, len_new, row_ptr_out, (int)n + 1, stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_degree_relabel (scan): %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    if (col_idx && col_out) {
        const int64_t nw = (n + 31) / 32;
        const int cgrid = (int)((nw + 7) / 8 < (int64_t)sms * 16 ? (nw + 7) / 8 : (int64_t)sms * 16);
        int32_t *dst = sort_rows ? (int32_t *)(w + L.off_cols) : col_out;
        relabel_copy_kernel<<<cgrid, RELABEL_THREADS, 0, stream>>>(n, order, row_ptr, col_idx, perm_out, row_ptr_out,
                                                                   dst, long_rows, ctr);
        relabel_long_kernel<<<sms, 1024, 0, stream>>>(order, row_ptr, col_idx, perm_out, row_ptr_out, dst,
                                                      long_rows, ctr);
        if (sort_rows) {
            tb = L.temp_bytes;
            e = cub::DeviceSegmentedSort::SortKeys(temp, tb, (const int32_t *)dst, col_out, (int)nnz, (int)n,
                                                   (const int32_t *)row_ptr_out, (const int32_t *)row_ptr_out + 1,
                                                   stream);
            if (e != cudaSuccess) {
                acsr_set_error("acsr_degree_relabel (row sort): %s", cudaGetErrorString(e));
                return ACSR_ERR_CUDA;
            }
        }
    }
    return acsr_check_launch("acsr_degree_relabel");
}

// ---------------------------------------------------------------------------------------
// acsr_permute_graph: rows reordered by `order` (new row i = old row order[i]) and every
// column mapped through col_map (NULL: kept) -- the same scan + copy kernels as the relabel.
namespace acsr {
__global__ void permute_len_kernel(int64_t n, const int32_t *__restrict__ order, const int32_t *__restrict__ rp,
                                   int32_t *__restrict__ len_new)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = order[i];
        len_new[i] = rp[u + 1] - rp[u];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) len_new[n] = 0;
}
}  // namespace acsr

extern "C" size_t acsr_permute_workspace_bytes(int64_t n) { return relabel_layout(n, 0, 0).total; }

extern "C" acsr_status acsr_permute_graph(int64_t n, const int32_t *row_ptr, const int32_t *col_idx,
                                          const int32_t *order, const int32_t *col_map, int32_t *row_ptr_out,
                                          int32_t *col_out, void *ws, size_t ws_bytes, cudaStream_t stream)
{
    if (n < 0 || n >= ((int64_t)1 << 31) - 1 || !row_ptr_out || (n > 0 && (!row_ptr || !order))) {
        acsr_set_error("acsr_permute_graph: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    const RelabelLayout L = relabel_layout(n, 0, 0);
    if (!ws || ws_bytes < L.total) {
        acsr_set_error("acsr_permute_graph: workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    if (n == 0) {
        cudaMemsetAsync(row_ptr_out, 0, sizeof(int32_t), stream);
        return acsr_check_launch("acsr_permute_graph");
    }
    char *w = (char *)ws;
    int32_t *len_new = (int32_t *)(w + L.off_len), *long_rows = (int32_t *)(w + L.off_long);
    int32_t *ctr = (int32_t *)(w + L.off_ctr);
    void *temp = w + L.off_temp;
    const int sms = acsr_num_sms();
    const int grid = (int)((n + RELABEL_THREADS - 1) / RELABEL_THREADS < (int64_t)sms * 8
                               ? (n + RELABEL_THREADS - 1) / RELABEL_THREADS : (int64_t)sms * 8);
    cudaMemsetAsync(ctr, 0, 16, stream);
    permute_len_kernel<<<grid, RELABEL_THREADS, 0, stream>>>(n, order, row_ptr, len_new);
    size_t tb = L.temp_bytes;
    const cudaError_t e = cub::DeviceScan::ExclusiveSum(temp, tb, len_new, row_ptr_out, (int)n + 1, stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_permute_graph (scan): %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    if (col_idx && col_out) {
        const int64_t nw = (n + 31) / 32;
        const int cgrid = (int)((nw + 7) / 8 < (int64_t)sms * 16 ? (nw + 7) / 8 : (int64_t)sms * 16);
        relabel_copy_kernel<<<cgrid, RELABEL_THREADS, 0, stream>>>(n, order, row_ptr, col_idx, col_map, row_ptr_out,
                                                                   col_out, long_rows, ctr);
        relabel_long_kernel<<<sms, 1024, 0, stream>>>(order, row_ptr, col_idx, col_map, row_ptr_out, col_out,
                                                      long_rows, ctr);
    }
    return acsr_check_launch("acsr_permute_graph");
}
