// tma_gather_bench.cu -- does the TMA engine (cp.async.bulk.tensor ... tile::gather4)
// give a random-gather path that beats the LSU path (~197 G gathers/s on an L2-resident
// x, tools/gather_bench.cu)?  y[i] = x[idx[i]]: x viewed as a 2-D tensor of 16-byte rows
// (2 doubles); every lane issues one gather4 (4 random rows -> 64 B of shared memory),
// a per-warp mbarrier collects the bytes, lanes pick their element and store y.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tma_gather_bench tools/tma_gather_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t s32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

constexpr int SLOT = 128;  // TMA destination must be 128-byte aligned (64 B used)

template <int STAGES, int NWARP>
__global__ void __launch_bounds__(NWARP * 32, 1) tma_gather(const __grid_constant__ CUtensorMap tmap,
                                                            const int *__restrict__ idx, double *__restrict__ y, long n)
{
    // per warp: STAGES x 32 lanes x SLOT B
    extern __shared__ unsigned char smem_raw[];
    unsigned char *smem = (unsigned char *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t bars[NWARP][STAGES];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned char *wbuf = smem + (size_t)warp * STAGES * 32 * SLOT;
    if (lane == 0)
        for (int s = 0; s < STAGES; s++) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&bars[warp][s])));
        }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    const long gw = (long)blockIdx.x * NWARP + warp, nw = (long)gridDim.x * NWARP;
    uint32_t phase[STAGES];
    for (int s = 0; s < STAGES; s++) phase[s] = 0;
    // each warp iteration handles 128 consecutive elements (4 per lane)
    long it = 0;
    int c[STAGES][4];
    long base[STAGES];
    auto issue = [&](int s, long b) {
        base[s] = b;
        const long i = b + 4 * lane;
        for (int k = 0; k < 4; k++) c[s][k] = (i + k < n) ? __ldcs(idx + i + k) : 0;
        if (lane == 0)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(&bars[warp][s])),
                         "r"(32 * 64) : "memory");
        __syncwarp();
        unsigned char *dst = wbuf + ((size_t)s * 32 + lane) * SLOT;
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(s32(dst)),
            "l"(&tmap), "r"(s32(&bars[warp][s])), "r"(0), "r"(c[s][0] >> 1), "r"(c[s][1] >> 1),
            "r"(c[s][2] >> 1), "r"(c[s][3] >> 1)
            : "memory");
    };
    auto drain = [&](int s) {
        uint32_t done = 0;
        while (!done)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                         : "=r"(done) : "r"(s32(&bars[warp][s])), "r"(phase[s]) : "memory");
        phase[s] ^= 1;
        const double *src = (const double *)(wbuf + ((size_t)s * 32 + lane) * SLOT);
        const long i = base[s] + 4 * lane;
        for (int k = 0; k < 4; k++)
            if (i + k < n) y[i + k] = src[2 * k + (c[s][k] & 1)];
        __syncwarp();
    };
    long b = gw * 128;
    int inflight = 0;
    for (int s = 0; s < STAGES && b < n; s++, b += nw * 128) { issue(s, b); inflight++; }
    int s = 0;
    while (inflight) {
        drain(s);
        inflight--;
        if (b < n) { issue(s, b); b += nw * 128; inflight++; }
        s = (s + 1) % STAGES;
        it++;
    }
}

// mixed: warps [0, NT) use TMA gather4 (1 stage), warps [NT, NWARP) use LSU gathers (ILP 4);
// work split by element ranges proportional to the warp counts
template <int NWARP, int NT>
__global__ void __launch_bounds__(NWARP * 32, 1) mixed_gather(const __grid_constant__ CUtensorMap tmap,
                                                              const double *__restrict__ x,
                                                              const int *__restrict__ idx, double *__restrict__ y,
                                                              long n, long split)
{
    extern __shared__ unsigned char smem_raw[];
    unsigned char *smem = (unsigned char *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ __align__(8) uint64_t bars[NT];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (warp < NT) {
        unsigned char *wbuf = smem + (size_t)warp * 32 * SLOT;
        if (lane == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&bars[warp])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        __syncwarp();
        uint32_t phase = 0;
        const long gw = (long)blockIdx.x * NT + warp, nw = (long)gridDim.x * NT;
        for (long b = gw * 128; b < split; b += nw * 128) {
            const long i = b + 4 * lane;
            int c[4];
            for (int k = 0; k < 4; k++) c[k] = (i + k < split) ? __ldcs(idx + i + k) : 0;
            if (lane == 0)
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(&bars[warp])),
                             "r"(32 * 64) : "memory");
            __syncwarp();
            unsigned char *dst = wbuf + (size_t)lane * SLOT;
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
                " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(s32(dst)),
                "l"(&tmap), "r"(s32(&bars[warp])), "r"(0), "r"(c[0] >> 1), "r"(c[1] >> 1), "r"(c[2] >> 1),
                "r"(c[3] >> 1)
                : "memory");
            uint32_t done = 0;
            while (!done)
                asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                             : "=r"(done) : "r"(s32(&bars[warp])), "r"(phase) : "memory");
            phase ^= 1;
            const double *src = (const double *)dst;
            for (int k = 0; k < 4; k++)
                if (i + k < split) y[i + k] = src[2 * k + (c[k] & 1)];
            __syncwarp();
        }
    } else {
        const int lw = warp - NT;
        const long gw = (long)blockIdx.x * (NWARP - NT) + lw, nw = (long)gridDim.x * (NWARP - NT);
        for (long b = split + gw * 128; b < n; b += nw * 128) {
            int c[4];
            double v[4];
            for (int k = 0; k < 4; k++) { long i = b + k * 32 + lane; c[k] = i < n ? __ldcs(idx + i) : 0; }
            for (int k = 0; k < 4; k++) v[k] = __ldg(x + c[k]);
            for (int k = 0; k < 4; k++) { long i = b + k * 32 + lane; if (i < n) y[i] = v[k]; }
        }
    }
}

typedef CUresult (*EncodeFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                             const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main(int argc, char **argv)
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long n = 16L << 20;
    std::vector<long> ncols_list = {1L << 20, 1L << 24, 1L << 26};
    int *idx;
    double *x, *y;
    CK(cudaMalloc(&idx, n * 4));
    CK(cudaMalloc(&y, n * 8));
    CK(cudaMalloc(&x, (1L << 26) * 8));
    std::vector<double> hx(1L << 20);
    for (long i = 0; i < (1L << 20); i++) hx[i] = (double)i;
    CK(cudaMemcpy(x, hx.data(), hx.size() * 8, cudaMemcpyHostToDevice));
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    EncodeFn encode = (EncodeFn)fn;
    std::vector<int> h(n);
    for (long ncols : ncols_list) {
        uint64_t s = 88172645463325252ull;
        for (long i = 0; i < n; i++) {
            s ^= s << 13; s ^= s >> 7; s ^= s << 17;
            h[i] = (int)(s % (uint64_t)ncols);
        }
        CK(cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice));
        CUtensorMap tmap;
        cuuint64_t dims[2] = {2, (cuuint64_t)(ncols / 2)};
        cuuint64_t strides[1] = {16};
        cuuint32_t box[2] = {2, 1};
        cuuint32_t estr[2] = {1, 1};
        CUresult r = encode(&tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, x, dims, strides, box, estr,
                            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) { printf("{\"error\": \"encode %d\"}\n", (int)r); return 1; }
        float ms = 0;
        auto runcfg = [&](auto kern, int nwarp, int stages) -> float {
            size_t smem = (size_t)nwarp * stages * 32 * SLOT + 1024;
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            for (int w = 0; w < 2; w++) kern<<<sms, nwarp * 32, smem>>>(tmap, idx, y, n);
            if (cudaDeviceSynchronize() != cudaSuccess) return -1.f;
            cudaEventRecord(a);
            for (int rr = 0; rr < 10; rr++) kern<<<sms, nwarp * 32, smem>>>(tmap, idx, y, n);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float t;
            cudaEventElapsedTime(&t, a, b);
            return t / 10;
        };
        const int STAGES = 0;
        float t1 = runcfg(tma_gather<2, 16>, 16, 2);
        float t2 = runcfg(tma_gather<3, 16>, 16, 3);
        float t3 = runcfg(tma_gather<6, 8>, 8, 6);
        float t4 = runcfg(tma_gather<1, 32>, 32, 1);
        printf("{\"ncols\": %ld, \"cfg\": \"16w x 2st\", \"Ggather_s\": %.1f}\n", ncols, n / (t1 * 1e-3) / 1e9);
        printf("{\"ncols\": %ld, \"cfg\": \"16w x 3st\", \"Ggather_s\": %.1f}\n", ncols, n / (t2 * 1e-3) / 1e9);
        printf("{\"ncols\": %ld, \"cfg\": \"8w x 6st\", \"Ggather_s\": %.1f}\n", ncols, n / (t3 * 1e-3) / 1e9);
        printf("{\"ncols\": %ld, \"cfg\": \"32w x 1st\", \"Ggather_s\": %.1f}\n", ncols, n / (t4 * 1e-3) / 1e9);
        ms = t2;
        CK(cudaGetLastError());
        for (double frac : {0.0, 0.25, 0.33, 0.4}) {
            long split = ((long)(n * frac) / 128) * 128;
            size_t smem = (size_t)16 * 32 * SLOT + 1024;
            auto k = mixed_gather<32, 16>;
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            k<<<sms, 1024, smem>>>(tmap, x, idx, y, n, split);
            CK(cudaDeviceSynchronize());
            cudaEventRecord(a);
            for (int rr = 0; rr < 10; rr++) k<<<sms, 1024, smem>>>(tmap, x, idx, y, n, split);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float t;
            cudaEventElapsedTime(&t, a, b);
            t /= 10;
            printf("{\"ncols\": %ld, \"cfg\": \"mixed 16 TMA warps + 16 LSU warps, TMA share %.2f\", \"Ggather_s\": %.1f}\n",
                   ncols, frac, n / (t * 1e-3) / 1e9);
        }
        // verify (first 1M cols hold i as value)
        bool ok = true;
        if (ncols == (1L << 20)) {
            std::vector<double> hy(n);
            CK(cudaMemcpy(hy.data(), y, n * 8, cudaMemcpyDeviceToHost));
            for (long i = 0; i < n; i += 997)
                if (hy[i] != (double)h[i]) { ok = false; break; }
        }
        printf("{\"ncols\": %ld, \"stages\": %d, \"us\": %.2f, \"Ggather_s\": %.1f, \"correct\": %s}\n", ncols, STAGES,
               ms * 1e3, n / (ms * 1e-3) / 1e9, ok ? "true" : "false");
    }
    return 0;
}
