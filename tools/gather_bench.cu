// gather_bench.cu -- calibrates the random-gather roofline of a B200: y[i] = x[idx[i]]
// with coalesced idx/y and random idx, and variants that tell the candidate limiters
// apart (every launch is error-checked; a failed configuration aborts the run):
//   mode 0 "gather8"   one random 8-byte x load per element (32 distinct lines per warp load)
//   mode 1 "pair8"     lanes 2i, 2i+1 read the two halves of one random 16-byte slot
//                      (16 distinct lines per warp load, 8 bytes per lane)
//   mode 2 "gather16"  one random 16-byte load (ld.v2.f64) per element (32 lines, 2x bytes)
//   mode 3 "gather32"  two 16-byte loads of one random 32-byte sector per element
//   mode 4 "stream"    coalesced 8-byte loads x[i] (no gather; request-rate reference)
// If the rate in gathers/s is the same for gather8 / gather16 / gather32, the limit is
// per request (L1TEX t-stage / miss path / LTS tag rate), not bytes; pair8 halves the
// distinct lines per warp load.
// Standalone (nvcc, no torch):
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -lineinfo -o gather_bench tools/gather_bench.cu
// Output: one JSON line per configuration.
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

template <int MODE, int ILP>
__global__ void __launch_bounds__(1024) gather(const int *__restrict__ idx, const double *__restrict__ x,
                                               double *__restrict__ y, long n)
{
    long base = ((long)blockIdx.x * blockDim.x) * ILP + threadIdx.x;
    const long stride = (long)gridDim.x * blockDim.x * ILP;
    const int lane = threadIdx.x & 31;
    for (; base < n; base += stride) {
        int c[ILP];
        double v[ILP];
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            const long i = base + (long)u * blockDim.x;
            c[u] = i < n ? __ldcs(idx + i) : 0;
        }
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            const long i = base + (long)u * blockDim.x;
            if (MODE == 0) {
                v[u] = __ldg(x + c[u]);
            } else if (MODE == 1) {
                const int cc = __shfl_sync(0xffffffffu, c[u], lane & ~1);
                v[u] = __ldg(x + ((cc & ~1) | (lane & 1)));
            } else if (MODE == 2) {
                const double2 p = __ldg((const double2 *)(x + (c[u] & ~1)));
                v[u] = p.x + p.y;
            } else if (MODE == 3) {
                const double2 *q = (const double2 *)(x + (c[u] & ~3));
                const double2 p0 = __ldg(q), p1 = __ldg(q + 1);
                v[u] = (p0.x + p0.y) + (p1.x + p1.y);
            } else {
                v[u] = __ldg(x + (i < n ? i : 0));
            }
        }
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            const long i = base + (long)u * blockDim.x;
            if (i < n) y[i] = v[u];
        }
    }
}

template <int MODE, int ILP>
static float run(const int *idx, const double *x, double *y, long n, int threads, int blocks_per_sm, int sms,
                 bool once)
{
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    const int grid = blocks_per_sm * sms;
    const int W = once ? 1 : 3, R = once ? 1 : 10;
    for (int w = 0; w < W; w++) gather<MODE, ILP><<<grid, threads>>>(idx, x, y, n);
    CK(cudaGetLastError());
    CK(cudaEventRecord(a));
    for (int r = 0; r < R; r++) gather<MODE, ILP><<<grid, threads>>>(idx, x, y, n);
    CK(cudaGetLastError());
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    CK(cudaGetLastError());
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    CK(cudaEventDestroy(a));
    CK(cudaEventDestroy(b));
    return ms / R;
}

static const char *mode_name(int m)
{
    static const char *s[] = {"gather8", "pair8", "gather16", "gather32", "stream"};
    return s[m];
}

int main(int argc, char **argv)
{
    // argv[1] == "ncu": one launch per mode at the C2 size (for a profiler pass)
    const bool ncu = argc > 1 && argv[1][0] == 'n';
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const long n = 16L << 20;
    std::vector<long> ncols_list = {1L << 20, 1L << 14, 1L << 17, 1L << 24, 1L << 26};
    if (ncu) ncols_list = {1L << 20};
    int *idx;
    double *x, *y;
    CK(cudaMalloc(&idx, n * 4));
    CK(cudaMalloc(&y, n * 8));
    CK(cudaMalloc(&x, (1L << 26) * 8 + 64));
    CK(cudaMemset(x, 0, (1L << 26) * 8 + 64));
    std::vector<int> h(n);
    for (long ncols : ncols_list) {
        uint64_t s = 88172645463325252ull;
        for (long i = 0; i < n; i++) {
            s ^= s << 13;
            s ^= s >> 7;
            s ^= s << 17;
            h[i] = (int)(s % (uint64_t)ncols);
        }
        CK(cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice));
        struct Cfg {
            int threads, bps;
        };
        const Cfg cfgs[] = {{1024, 2}, {256, 8}, {512, 4}};
        for (const Cfg cf : cfgs) {
            if (ncu && cf.threads != 1024) continue;
            float t[5][3];
            t[0][0] = run<0, 4>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[1][0] = run<1, 4>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[2][0] = run<2, 4>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[3][0] = run<3, 4>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[4][0] = run<4, 4>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[0][1] = run<0, 8>(idx, x, y, n, cf.threads, cf.bps, sms, ncu);
            t[0][2] = cf.threads <= 512 ? run<0, 16>(idx, x, y, n, cf.threads, cf.bps, sms, ncu) : -1.f;
            for (int m = 0; m < 5; m++)
                printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"mode\": \"%s\", \"ilp\": 4, "
                       "\"us\": %.2f, \"Ggather_s\": %.1f}\n",
                       ncols, cf.threads, cf.bps, mode_name(m), t[m][0] * 1e3, n / (t[m][0] * 1e-3) / 1e9);
            printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"mode\": \"gather8\", \"ilp\": 8, "
                   "\"us\": %.2f, \"Ggather_s\": %.1f}\n",
                   ncols, cf.threads, cf.bps, t[0][1] * 1e3, n / (t[0][1] * 1e-3) / 1e9);
            if (t[0][2] > 0)
                printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"mode\": \"gather8\", \"ilp\": 16, "
                       "\"us\": %.2f, \"Ggather_s\": %.1f}\n",
                       ncols, cf.threads, cf.bps, t[0][2] * 1e3, n / (t[0][2] * 1e-3) / 1e9);
            fflush(stdout);
        }
    }
    return 0;
}
