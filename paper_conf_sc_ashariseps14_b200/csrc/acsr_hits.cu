// acsr_hits.cu -- HITS normalisation (Eq. 5-7; reading R6): after the
// block SpMV y = [[0, A^T], [A, 0]] [a; h], scale each half to unit Euclidean norm and
// measure the distance to the previous iterate.  Two small launches, fixed grid and
// fixed reduction order (per-CTA tree + last-CTA ordered sum) -> deterministic.
#include <cuda_runtime.h>

#include "acsr_internal.cuh"

namespace acsr {

constexpr int HITS_THREADS = 256;
constexpr int HITS_CTAS = 296;  // 2 x 148 SMs; fixed so the reduction order is fixed

struct HitsWs {
    double part[2][HITS_CTAS];
    double norm[2];
    int ticket;
};

__device__ __forceinline__ double block_sum(double v, double *sh)
{
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (lane == 0) sh[w] = v;
    __syncthreads();
    double t = 0.0;
    if (threadIdx.x == 0)
        for (int i = 0; i < HITS_THREADS / 32; i++) t += sh[i];
    __syncthreads();
    return t;  // valid in thread 0
}

// mode 0: sums of y^2 per half -> norms;  mode 1: v_next = y / norm, sums of (v_next - v)^2
__global__ void __launch_bounds__(HITS_THREADS) hits_kernel(int64_t n, const double *__restrict__ y,
                                                            const double *__restrict__ v,
                                                            double *__restrict__ vn, HitsWs *ws,
                                                            double *dist2, int mode, int32_t *ctrl, double eps2)
{
    __shared__ double sh[HITS_THREADS / 32];
    __shared__ int last;
    if (ctrl && *(volatile int32_t *)ctrl) return;  // converged earlier: no-op (device-side loop)
    double acc[2] = {0.0, 0.0};
    const double na = mode ? ws->norm[0] : 0.0, nh = mode ? ws->norm[1] : 0.0;
    for (int64_t i = blockIdx.x * (int64_t)HITS_THREADS + threadIdx.x; i < 2 * n;
         i += (int64_t)HITS_CTAS * HITS_THREADS) {
        const int half = i >= n;
        const double yi = y[i];
        if (mode == 0) {
            acc[half] = fma(yi, yi, acc[half]);
        } else {
            const double nm = half ? nh : na;
            const double t = nm > 0.0 ? yi / nm : 0.0;
            vn[i] = t;
            const double d = t - v[i];
            acc[half] = fma(d, d, acc[half]);
        }
    }
    for (int h = 0; h < 2; h++) {
        const double t = block_sum(acc[h], sh);
        if (threadIdx.x == 0) ws->part[h][blockIdx.x] = t;
    }
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(&ws->ticket, 1) == HITS_CTAS - 1;
    }
    __syncthreads();
    if (last && threadIdx.x < 2) {
        __threadfence();
        double t = 0.0;
        for (int b = 0; b < HITS_CTAS; b++) t += __ldcg(&ws->part[threadIdx.x][b]);
        if (mode == 0) ws->norm[threadIdx.x] = sqrt(t);
        else dist2[threadIdx.x] = t;
        const double th = __shfl_sync(0x3u, t, 1);  // the hub distance (thread 1)
        if (threadIdx.x == 0 && mode == 1 && ctrl) {
            ctrl[1] += 1;
            // both Euclidean distances <= eps ("until both ... converge")
            if (t <= eps2 && th <= eps2) ctrl[0] = 1;
        }
    }
    if (last && threadIdx.x == 0) ws->ticket = 0;
}

}  // namespace acsr

using namespace acsr;

extern "C" size_t acsr_hits_workspace_bytes(int64_t n)
{
    (void)n;
    return align_up(sizeof(HitsWs), 256);
}

extern "C" acsr_status acsr_hits_normalize(int64_t n, const double *y, const double *v, double *v_next,
                                           double *dist2, void *ws, size_t ws_bytes, cudaStream_t stream)
{
    return acsr_hits_normalize_ctrl(n, y, v, v_next, dist2, nullptr, -1.0, ws, ws_bytes, stream);
}

extern "C" acsr_status acsr_hits_normalize_ctrl(int64_t n, const double *y, const double *v, double *v_next,
                                                double *dist2, int32_t *ctrl, double eps2, void *ws, size_t ws_bytes,
                                                cudaStream_t stream)
{
    if (n < 0 || !dist2 || (n > 0 && (!y || !v || !v_next))) {
        acsr_set_error("acsr_hits_normalize: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (!ws || ws_bytes < acsr_hits_workspace_bytes(n)) {
        acsr_set_error("acsr_hits_normalize: workspace too small");
        return ACSR_ERR_WORKSPACE;
    }
    HitsWs *w = (HitsWs *)ws;
    cudaMemsetAsync(&w->ticket, 0, sizeof(int), stream);
    hits_kernel<<<HITS_CTAS, HITS_THREADS, 0, stream>>>(n, y, v, v_next, w, dist2, 0, ctrl, eps2);
    hits_kernel<<<HITS_CTAS, HITS_THREADS, 0, stream>>>(n, y, v, v_next, w, dist2, 1, ctrl, eps2);
    return acsr_check_launch("acsr_hits_normalize");
}
