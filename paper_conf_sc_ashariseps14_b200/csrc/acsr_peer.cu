// acsr_peer.cu -- the multi-GPU PageRank exchange (A9 of SURVEY §8(a)) fused into the
// step over peer memory (NEXT N1; §8(e) lever 1).
//
// Row-partitioned PageRank (§VIII, reading Q19) needs, after every step, each
// rank's slice of xs' = x'/outdeg in every rank's replicated xs.  Instead of a separate
// all-gather after the step, each rank's fused step kernel (acsr_spmv.cu, PR path) stores
// every finished slice entry straight into all ranks' xs buffers -- NVLink/NVSwitch P2P
// stores issued while the rest of the step is still running -- and its last CTA
// publishes the push (Delta^2 partial + a release flag) to every rank.  The next step
// waits on the flags at entry instead of a host-side collective.
//
// Memory: one library-owned region per rank (PeerState + two xs buffers, alternating by
// push parity), exported with cudaIpcGetMemHandle and mapped by every other rank with
// cudaIpcOpenMemHandle (same node; NVLink P2P between GPUs, or plain device memory when
// several ranks share one GPU).  The handle exchange itself is the caller's (host bytes,
// e.g. torch.distributed.all_gather_object).
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>

#include <new>

#include "acsr_internal.cuh"

namespace acsr {

// xs slice of the initial / warm-start iterate: xs = x / outdeg (IEEE division, as
// acsr_pagerank_scale) for the local rows, rows < slice_len pushed to every rank.
__global__ void peer_push_kernel(int64_t n, const double *__restrict__ x, const int32_t *__restrict__ outdeg,
                                 double *__restrict__ xs_local, PeerArgs p)
{
    __shared__ unsigned long long s_c;
    if (threadIdx.x == 0) {
        const unsigned long long c = *(volatile unsigned long long *)&p.st->pushes;
        peer_wait(p, c);  // every rank is done reading the buffer this push overwrites
        s_c = c;
    }
    __syncthreads();
    const unsigned long long c = s_c;
    const int64_t off = p.off_buf[c & 1];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int od = outdeg[i];
        const double v = od > 0 ? x[i] / (double)od : 0.0;
        if (xs_local) xs_local[i] = v;
        if (i < p.slice_len)
            for (int q = 0; q < p.nranks; q++) *(double *)(p.base[q] + off + 8 * (p.slice_off + i)) = v;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();
        if (atomicAdd(&p.st->ticket, 1u) == gridDim.x - 1) {
            __threadfence_system();
            p.st->ticket = 0;
            peer_signal(p, c + 1, false, 0, 0, 0);
        }
    }
}

// Global Delta^2 of the last push: wait for every rank's push, add the fixed-point
// partials (exact, so every rank gets the same bits whatever the order), and set the
// device-side stop flag.  ctrl[0] already set: converged earlier, nothing to do.
__global__ void peer_delta2_kernel(PeerArgs p, double *delta2, int32_t *ctrl, double eps2)
{
    if (threadIdx.x != 0) return;
    if (ctrl && *(volatile int32_t *)ctrl) return;
    const unsigned long long c = *(volatile unsigned long long *)&p.st->pushes;
    peer_wait(p, c);
    const double d2v = p.st->last_step ? peer_sum_d2(p, c) : 0.0;
    *delta2 = d2v;
    if (ctrl && d2v <= eps2) ctrl[0] = 1;
}

}  // namespace acsr

using namespace acsr;

static int64_t buf_off(int which, int64_t xs_len)
{
    const int64_t b0 = (int64_t)align_up(sizeof(PeerState), PEER_BUF_ALIGN);
    return which == 0 ? b0 : b0 + (int64_t)align_up(sizeof(double) * (size_t)xs_len, PEER_BUF_ALIGN);
}

extern "C" acsr_status acsr_peer_create(acsr_peer **out, int nranks, int rank, int64_t xs_len, int64_t slice_off,
                                        int64_t slice_len, void *handle)
{
    if (!out || !handle || nranks < 1 || nranks > ACSR_PEER_MAX || rank < 0 || rank >= nranks || xs_len < 0 ||
        slice_off < 0 || slice_len < 0 || slice_off + slice_len > xs_len) {
        acsr_set_error("acsr_peer_create: invalid argument (1 <= nranks <= %d, 0 <= rank < nranks, "
                       "slice inside [0, xs_len))", ACSR_PEER_MAX);
        return ACSR_ERR_INVALID_VALUE;
    }
    *out = nullptr;
    acsr_peer *p = new (std::nothrow) acsr_peer();
    if (!p) return ACSR_ERR_CUDA;
    p->nranks = nranks;
    p->rank = rank;
    p->xs_len = xs_len;
    p->slice_off = slice_off;
    p->slice_len = slice_len;
    cudaGetDevice(&p->device);
    p->bytes = (size_t)buf_off(1, xs_len) + align_up(sizeof(double) * (size_t)xs_len, PEER_BUF_ALIGN);
    cudaError_t e = cudaMalloc(&p->region, p->bytes);
    if (e == cudaSuccess) e = cudaMemset(p->region, 0, p->bytes);  // flags 0, buffers +0.0
    cudaIpcMemHandle_t h;
    if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, p->region);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        acsr_set_error("acsr_peer_create: %s", cudaGetErrorString(e));
        if (p->region) cudaFree(p->region);
        delete p;
        return ACSR_ERR_CUDA;
    }
    static_assert(sizeof(cudaIpcMemHandle_t) <= ACSR_IPC_HANDLE_BYTES, "IPC handle size");
    memset(handle, 0, ACSR_IPC_HANDLE_BYTES);
    memcpy(handle, &h, sizeof(h));
    *out = p;
    return ACSR_OK;
}

extern "C" acsr_status acsr_peer_open(acsr_peer *p, const void *handles)
{
    if (!p || !handles || p->opened) {
        acsr_set_error("acsr_peer_open: invalid argument (NULL, or already opened)");
        return ACSR_ERR_INVALID_VALUE;
    }
    PeerArgs a{};
    a.nranks = p->nranks;
    a.rank = p->rank;
    a.off_buf[0] = buf_off(0, p->xs_len);
    a.off_buf[1] = buf_off(1, p->xs_len);
    a.slice_off = p->slice_off;
    a.slice_len = p->slice_len;
    a.xs_len = p->xs_len;
    {
        const char *e = getenv("ACSR_PEER_TIMEOUT_MS");
        const long long ms = (e && e[0]) ? atoll(e) : 20000;
        a.timeout_ns = (unsigned long long)(ms > 0 ? ms : 20000) * 1000000ull;
    }
    for (int q = 0; q < p->nranks; q++) {
        if (q == p->rank) {
            a.base[q] = p->region;
            continue;
        }
        cudaIpcMemHandle_t h;
        memcpy(&h, (const char *)handles + (size_t)q * ACSR_IPC_HANDLE_BYTES, sizeof(h));
        void *ptr = nullptr;
        const cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            acsr_set_error("acsr_peer_open: rank %d: %s", q, cudaGetErrorString(e));
            for (int j = 0; j < q; j++)
                if (j != p->rank) cudaIpcCloseMemHandle(a.base[j]);
            return ACSR_ERR_CUDA;
        }
        a.base[q] = (char *)ptr;
    }
    a.st = (PeerState *)p->region;
    const cudaError_t e = cudaMemcpy((char *)p->region + offsetof(PeerState, view), &a, sizeof(a),
                                     cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_peer_open: %s", cudaGetErrorString(e));
        for (int j = 0; j < p->nranks; j++)
            if (j != p->rank) cudaIpcCloseMemHandle(a.base[j]);
        return ACSR_ERR_CUDA;
    }
    p->args = a;
    p->opened = true;
    return ACSR_OK;
}

extern "C" acsr_status acsr_peer_destroy(acsr_peer *p)
{
    if (!p) return ACSR_OK;
    cudaError_t e = cudaDeviceSynchronize();
    if (p->opened)
        for (int q = 0; q < p->nranks; q++)
            if (q != p->rank && p->args.base[q]) cudaIpcCloseMemHandle(p->args.base[q]);
    if (p->region) cudaFree(p->region);
    delete p;
    if (e != cudaSuccess) {
        acsr_set_error("acsr_peer_destroy: %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    return ACSR_OK;
}

extern "C" acsr_status acsr_peer_push(acsr_peer *p, int64_t n, const double *x, const int32_t *outdeg,
                                      double *xs_local, cudaStream_t stream)
{
    if (!p || !p->opened || n < p->slice_len || (n > 0 && (!x || !outdeg))) {
        acsr_set_error("acsr_peer_push: invalid argument (opened peer, n >= slice_len)");
        return ACSR_ERR_INVALID_VALUE;
    }
    int64_t blocks = (n + 255) / 256;
    if (blocks > (int64_t)acsr_num_sms() * 8) blocks = (int64_t)acsr_num_sms() * 8;
    if (blocks < 1) blocks = 1;
    peer_push_kernel<<<(int)blocks, 256, 0, stream>>>(n, x, outdeg, xs_local, p->args);
    return acsr_check_launch("acsr_peer_push");
}

extern "C" acsr_status acsr_peer_delta2(acsr_peer *p, double *delta2, int32_t *ctrl, double eps2,
                                        cudaStream_t stream)
{
    if (!p || !p->opened || !delta2) {
        acsr_set_error("acsr_peer_delta2: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    peer_delta2_kernel<<<1, 32, 0, stream>>>(p->args, delta2, ctrl, eps2);
    return acsr_check_launch("acsr_peer_delta2");
}

extern "C" acsr_status acsr_peer_query(const acsr_peer *p, int64_t *pushes, int32_t *error,
                                       const double **xs_current)
{
    if (!p) {
        acsr_set_error("acsr_peer_query: NULL peer");
        return ACSR_ERR_INVALID_VALUE;
    }
    PeerState st;
    const cudaError_t e = cudaMemcpy(&st, p->region, sizeof(st), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) {
        acsr_set_error("acsr_peer_query: %s", cudaGetErrorString(e));
        return ACSR_ERR_CUDA;
    }
    if (pushes) *pushes = (int64_t)st.pushes;
    if (error) *error = (int32_t)st.err;
    if (xs_current)
        *xs_current = st.pushes ? (const double *)(p->region + buf_off((int)((st.pushes + 1) & 1), p->xs_len)) : nullptr;
    return ACSR_OK;
}

// dst[0 .. xs_len) = the local buffer holding the last push (the parity is read on the
// device, so the copy is stream-ordered after the push); zeros before the first push
__global__ void peer_read_kernel(const PeerArgs *v, double *dst)
{
    const unsigned long long c = *(volatile unsigned long long *)&v->st->pushes;
    const double *src = (const double *)(v->base[v->rank] + v->off_buf[(c + 1) & 1]);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < v->xs_len; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = c ? src[i] : 0.0;
}

extern "C" acsr_status acsr_peer_read_xs(const acsr_peer *p, double *dst, cudaStream_t stream)
{
    if (!p || !p->opened || (p->xs_len > 0 && !dst)) {
        acsr_set_error("acsr_peer_read_xs: invalid argument");
        return ACSR_ERR_INVALID_VALUE;
    }
    if (p->xs_len == 0) return ACSR_OK;
    int64_t blocks = (p->xs_len + 255) / 256;
    if (blocks > (int64_t)acsr_num_sms() * 8) blocks = (int64_t)acsr_num_sms() * 8;
    peer_read_kernel<<<(int)blocks, 256, 0, stream>>>(&((const PeerState *)p->region)->view, dst);
    return acsr_check_launch("acsr_peer_read_xs");
}
