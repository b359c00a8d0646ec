// acsr_grow.cu -- the grown slack-CSR layout of reading R4 (after a CAPACITY rejection of
// an update batch, §VII P:334 keeps "some additional memory ... at the end of each CSR
// row"; what happens when a row outgrows it is unstated): new capacities and their
// exclusive prefix on the device (CUB scan), so no planning arithmetic runs in Python.
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>

#include "acsr_internal.cuh"

namespace acsr {

__global__ void grow_caps_kernel(int64_t n, const int32_t *__restrict__ rb, const int32_t *__restrict__ re,
                                 const int32_t *__restrict__ cap, int32_t min_slack, int32_t frac,
                                 int64_t *__restrict__ cap64)
{
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t len = (int64_t)re[r] - rb[r];
        const int64_t c = cap[r];
        const int64_t gc = (c + frac - 1) / frac, gl = (len + frac - 1) / frac;
        const int64_t a = c + (gc > min_slack ? gc : min_slack);
        const int64_t b = len + (gl > min_slack ? gl : min_slack);
        cap64[r] = a > b ? a : b;
    }
}

__global__ void grow_write_kernel(int64_t n, const int64_t *__restrict__ cap64, const int64_t *__restrict__ pre,
                                  int32_t *__restrict__ new_begin, int32_t *__restrict__ new_cap, int64_t *total)
{
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        new_begin[r] = (int32_t)pre[r];
        new_cap[r] = (int32_t)cap64[r];
        if (r == n - 1) *total = pre[r] + cap64[r];
    }
}

}  // namespace acsr

using namespace acsr;

extern "C" size_t acsr_grow_workspace_bytes(int64_t n_rows)
{
    const size_t nn = (size_t)(n_rows > 0 ? n_rows : 1);
    size_t temp = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, temp, (const int64_t *)nullptr, (int64_t *)nullptr, (int)nn);
    return 2 * align_up(8 * nn, 256) + align_up(temp, 256);
}

extern "C" acsr_status acsr_grow_layout(int64_t n_rows, const int32_t *row_begin, const int32_t *row_end,
                                        const int32_t *row_cap, int32_t min_slack, int32_t frac, int32_t *new_begin,
                                        int32_t *new_cap, int64_t *total, void *ws, size_t ws_bytes,
                                        cudaStream_t stream)
{
    if (n_rows < 0 || n_rows >= ((int64_t)1 << 31) || min_slack < 1 || frac < 1 || !total ||
        (n_rows > 0 && (!row_begin || !row_end || !row_cap || !new_begin || !new_cap))) {
        acsr_set_error("acsr_grow_layout: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!ws || ws_bytes < acsr_grow_workspace_bytes(n_rows)) {
        acsr_set_error("acsr_grow_layout: workspace missing or too small");
        return ACSR_ERR_WORKSPACE;
    }
    if (n_rows == 0) {
        cudaMemsetAsync(total, 0, sizeof(int64_t), stream);
        return acsr_check_launch("acsr_grow_layout");
    }
    const size_t nn = (size_t)n_rows;
    int64_t *cap64 = (int64_t *)ws;
    int64_t *pre = (int64_t *)((char *)ws + align_up(8 * nn, 256));
    void *temp = (char *)ws + 2 * align_up(8 * nn, 256);
    size_t tb = ws_bytes - 2 * align_up(8 * nn, 256);
    const int sms = acsr_num_sms();
    const int grid = (int)((n_rows + 255) / 256 < (int64_t)sms * 8 ? (n_rows + 255) / 256 : (int64_t)sms * 8);
    grow_caps_kernel<<<grid, 256, 0, stream>>>(n_rows, row_begin, row_end, row_cap, min_slack, frac, cap64);
    const cudaError_t e = cub::DeviceScan::ExclusiveSum(temp, tb, cap64, pre, (int)n_rows, stream);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_grow_layout (scan): %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    grow_write_kernel<<<grid, 256, 0, stream>>>(n_rows, cap64, pre, new_begin, new_cap, total);
    return acsr_check_launch("acsr_grow_layout");
}
