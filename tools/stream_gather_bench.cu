// stream_gather_bench.cu -- does streaming the CSR arrays through the LSU cost the random
// x gathers their throughput, and does moving the stream to TMA (cp.async.bulk into shared
// memory) give it back?  A synthetic SpMV-shaped kernel over nnz elements:
//   y[i / 32] = sum over a 32-element group of val[i] * x[col[i]]
// col/val are streamed (coalesced, DRAM), x (8 MB) is gathered at random (L2).
//   mode 0 "lsu":  col/val by 128-bit LDG (4 elements per lane, 8 gathers in flight)
//   mode 1 "tma":  col/val by per-warp double-buffered cp.async.bulk into shared memory,
//                  then LDS; the same gathers
//   mode 2 "gather_only": col by LDG, no val (the gather-bench reference)
// Standalone: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -lineinfo -o stream_gather_bench tools/stream_gather_bench.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>
#include <vector>

#define CK(x)                                                                                        \
    do {                                                                                             \
        cudaError_t e = (x);                                                                         \
        if (e != cudaSuccess) {                                                                      \
            fprintf(stderr, "CUDA error %s at line %d\n", cudaGetErrorString(e), __LINE__);          \
            exit(1);                                                                                 \
        }                                                                                            \
    } while (0)

constexpr int WARPS = 32;            // 1024-thread CTAs, one per SM
constexpr int CHUNK = 256;           // elements per warp iteration (8 per lane)
constexpr int STAGES = 2;

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(1024, 1) k_lsu(const int *__restrict__ col, const double *__restrict__ val,
                                                 const double *__restrict__ x, double *__restrict__ y, long nnz,
                                                 int with_val)
{
    const int lane = threadIdx.x & 31;
    const long w = (long)blockIdx.x * WARPS + (threadIdx.x >> 5), nw = (long)gridDim.x * WARPS;
    for (long base = w * CHUNK; base < nnz; base += nw * CHUNK) {
        const long e0 = base + 4 * lane, e1 = e0 + 128;
        const int4 c0 = __ldcs((const int4 *)(col + e0));
        const int4 c1 = __ldcs((const int4 *)(col + e1));
        double v[8] = {1, 1, 1, 1, 1, 1, 1, 1};
        if (with_val) {
            const double2 p0 = __ldcs((const double2 *)(val + e0)), p1 = __ldcs((const double2 *)(val + e0 + 2));
            const double2 p2 = __ldcs((const double2 *)(val + e1)), p3 = __ldcs((const double2 *)(val + e1 + 2));
            v[0] = p0.x; v[1] = p0.y; v[2] = p1.x; v[3] = p1.y; v[4] = p2.x; v[5] = p2.y; v[6] = p3.x; v[7] = p3.y;
        }
        double s = v[0] * __ldg(x + c0.x) + v[1] * __ldg(x + c0.y) + v[2] * __ldg(x + c0.z) + v[3] * __ldg(x + c0.w) +
                   v[4] * __ldg(x + c1.x) + v[5] * __ldg(x + c1.y) + v[6] * __ldg(x + c1.z) + v[7] * __ldg(x + c1.w);
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0) y[base / CHUNK] = s;
    }
}

__global__ void __launch_bounds__(1024, 1) k_tma(const int *__restrict__ col, const double *__restrict__ val,
                                                 const double *__restrict__ x, double *__restrict__ y, long nnz)
{
    // per warp: STAGES x (CHUNK ints + CHUNK doubles) = 2 x 3 KB; 32 warps = 192 KB
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ __align__(8) uint64_t bar[WARPS][STAGES];
    const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
    unsigned char *mine = sm + (size_t)wi * STAGES * CHUNK * 12;
    const long w = (long)blockIdx.x * WARPS + wi, nw = (long)gridDim.x * WARPS;
    if (lane == 0)
        for (int s = 0; s < STAGES; s++) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[wi][s])));
        }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    auto issue = [&](long base, int s) {
        if (lane == 0 && base < nnz) {
            int *dc = (int *)(mine + (size_t)s * CHUNK * 12);
            double *dv = (double *)(dc + CHUNK);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[wi][s])),
                         "r"(CHUNK * 12)
                         : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(dc)),
                         "l"(col + base), "r"(CHUNK * 4), "r"(smem_u32(&bar[wi][s]))
                         : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             smem_u32(dv)),
                         "l"(val + base), "r"(CHUNK * 8), "r"(smem_u32(&bar[wi][s]))
                         : "memory");
        }
    };
    uint32_t phase[STAGES] = {0, 0};
    long base = w * CHUNK;
    for (int s = 0; s < STAGES; s++) issue(base + (long)s * nw * CHUNK, s);
    int s = 0;
    for (; base < nnz; base += nw * CHUNK) {
        uint32_t done = 0;
        while (!done)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(done)
                         : "r"(smem_u32(&bar[wi][s])), "r"(phase[s])
                         : "memory");
        phase[s] ^= 1;
        const int *dc = (const int *)(mine + (size_t)s * CHUNK * 12);
        const double *dv = (const double *)(dc + CHUNK);
        const int4 c0 = ((const int4 *)dc)[lane], c1 = ((const int4 *)dc)[lane + 32];
        const double2 p0 = ((const double2 *)dv)[2 * lane], p1 = ((const double2 *)dv)[2 * lane + 1];
        const double2 p2 = ((const double2 *)dv)[64 + 2 * lane], p3 = ((const double2 *)dv)[64 + 2 * lane + 1];
        __syncwarp();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic reads before the async-proxy refill
        issue(base + (long)STAGES * nw * CHUNK, s);  // the stage is consumed (values in registers)
        double sacc = p0.x * __ldg(x + c0.x) + p0.y * __ldg(x + c0.y) + p1.x * __ldg(x + c0.z) + p1.y * __ldg(x + c0.w) +
                      p2.x * __ldg(x + c1.x) + p2.y * __ldg(x + c1.y) + p3.x * __ldg(x + c1.z) + p3.y * __ldg(x + c1.w);
        for (int o = 16; o > 0; o >>= 1) sacc += __shfl_xor_sync(0xffffffffu, sacc, o);
        if (lane == 0) y[base / CHUNK] = sacc;
        s = (s + 1) % STAGES;
    }
}

int main(int argc, char **argv)
{
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const long nnz = 16L << 20;  // C2-sized: 16.8 M non-zeros
    const long ncols = argc > 1 ? atol(argv[1]) : (1L << 20);
    int *col;
    double *val, *x, *y;
    CK(cudaMalloc(&col, nnz * 4));
    CK(cudaMalloc(&val, nnz * 8));
    CK(cudaMalloc(&x, ncols * 8));
    CK(cudaMalloc(&y, nnz / CHUNK * 8 + 8));
    CK(cudaMemset(val, 0, nnz * 8));
    CK(cudaMemset(x, 0, ncols * 8));
    std::vector<int> h(nnz);
    uint64_t s = 88172645463325252ull;
    for (long i = 0; i < nnz; i++) {
        s ^= s << 13;
        s ^= s >> 7;
        s ^= s << 17;
        h[i] = (int)(s % (uint64_t)ncols);
    }
    CK(cudaMemcpy(col, h.data(), nnz * 4, cudaMemcpyHostToDevice));
    char *flush;
    CK(cudaMalloc(&flush, 256 << 20));
    const size_t tma_smem = (size_t)WARPS * STAGES * CHUNK * 12;
    CK(cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tma_smem));
    const char *names[] = {"lsu", "tma", "gather_only"};
    for (int mode = 0; mode < 3; mode++) {
        float best = 1e30f, sum = 0.f;
        const int R = 10;
        for (int r = 0; r < R + 2; r++) {
            CK(cudaMemset(flush, r, 256 << 20));
            cudaEvent_t a, b;
            CK(cudaEventCreate(&a));
            CK(cudaEventCreate(&b));
            CK(cudaEventRecord(a));
            if (mode == 0) k_lsu<<<sms, 1024>>>(col, val, x, y, nnz, 1);
            else if (mode == 1) k_tma<<<sms, 1024, tma_smem>>>(col, val, x, y, nnz);
            else k_lsu<<<sms, 1024>>>(col, val, x, y, nnz, 0);
            CK(cudaGetLastError());
            CK(cudaEventRecord(b));
            CK(cudaEventSynchronize(b));
            float ms;
            CK(cudaEventElapsedTime(&ms, a, b));
            if (r >= 2) {
                best = ms < best ? ms : best;
                sum += ms;
            }
        }
        printf("{\"mode\": \"%s\", \"ncols\": %ld, \"nnz\": %ld, \"us_mean\": %.2f, \"us_min\": %.2f, \"Gnnz_s\": %.1f}\n",
               names[mode], ncols, nnz, sum / R * 1e3, best * 1e3, nnz / (sum / R * 1e-3) / 1e9);
        fflush(stdout);
    }
    return 0;
}
