// gather_bench.cu -- calibrates the random-gather roofline of a B200: y[i] = x[idx[i]]
// with coalesced idx/y and random idx over an L2-resident x, for several load flavours,
// loads in flight per thread (ILP) and block shapes.  Standalone (nvcc, no torch):
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o gather_bench tools/gather_bench.cu
// Output: one JSON line per configuration (G gathers/s, effective GB/s of 8-byte values).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s at %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

template <int FLAVOR>
__device__ __forceinline__ double ldx(const double *p)
{
    double v;
    if (FLAVOR == 0) v = *p;                  // default (ld.global / .ca)
    else if (FLAVOR == 1) v = __ldg(p);       // ld.global.nc
    else if (FLAVOR == 2) v = __ldcg(p);      // ld.global.cg (L2 only)
    else if (FLAVOR == 3) {                   // ld.global.nc.L1::no_allocate
        asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    } else {                                  // ld.global.L1::evict_last
        asm volatile("ld.global.L1::evict_last.f64 %0, [%1];" : "=d"(v) : "l"(p));
    }
    return v;
}

template <int FLAVOR, int ILP>
__global__ void gather(const int *__restrict__ idx, const double *__restrict__ x, double *__restrict__ y,
                       long n)
{
    long base = ((long)blockIdx.x * blockDim.x) * ILP + threadIdx.x;
    long stride = (long)gridDim.x * blockDim.x * ILP;
    for (; base < n; base += stride) {
        int c[ILP];
        double v[ILP];
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            long i = base + (long)u * blockDim.x;
            c[u] = i < n ? __ldcs(idx + i) : 0;
        }
#pragma unroll
        for (int u = 0; u < ILP; u++) v[u] = ldx<FLAVOR>(x + c[u]);
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            long i = base + (long)u * blockDim.x;
            if (i < n) y[i] = v[u];
        }
    }
}

template <int FLAVOR, int ILP>
static float run(const int *idx, const double *x, double *y, long n, int threads, int blocks_per_sm, int sms)
{
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int grid = blocks_per_sm * sms;
    for (int w = 0; w < 3; w++) gather<FLAVOR, ILP><<<grid, threads>>>(idx, x, y, n);
    cudaEventRecord(a);
    const int R = 10;
    for (int r = 0; r < R; r++) gather<FLAVOR, ILP><<<grid, threads>>>(idx, x, y, n);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / R;
}

int main(int argc, char **argv)
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long n = 16L << 20;
    std::vector<long> ncols_list = {1L << 20, 1L << 17, 1L << 14, 1L << 26, 1L << 24};
    if (argc > 1) ncols_list = {1L << 26, 1L << 24, 1L << 22};
    int *idx;
    double *x, *y;
    CK(cudaMalloc(&idx, n * 4));
    CK(cudaMalloc(&y, n * 8));
    CK(cudaMalloc(&x, (1L << 26) * 8));
    CK(cudaMemset(x, 0, (1L << 26) * 8));
    std::vector<int> h(n);
    for (long ncols : ncols_list) {
        uint64_t s = 88172645463325252ull;
        for (long i = 0; i < n; i++) {
            s ^= s << 13; s ^= s >> 7; s ^= s << 17;
            h[i] = (int)(s % (uint64_t)ncols);
        }
        CK(cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice));
        struct Cfg { int threads, bps; };
        Cfg cfgs[] = {{256, 8}, {1024, 2}, {512, 4}, {256, 4}};
        for (Cfg cf : cfgs) {
            float t[5][3];
            t[0][0] = run<0, 4>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[1][0] = run<1, 4>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[2][0] = run<2, 4>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[3][0] = run<3, 4>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[4][0] = run<4, 4>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[0][1] = run<1, 8>(idx, x, y, n, cf.threads, cf.bps, sms);
            t[0][2] = run<1, 16>(idx, x, y, n, cf.threads, cf.bps, sms);
            const char *names[5] = {"default", "nc", "cg", "nc_noalloc", "evict_last"};
            for (int f = 0; f < 5; f++)
                printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"flavor\": \"%s\", \"ilp\": 4, "
                       "\"us\": %.2f, \"Ggather_s\": %.1f}\n", ncols, cf.threads, cf.bps, names[f], t[f][0] * 1e3,
                       n / (t[f][0] * 1e-3) / 1e9);
            printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"flavor\": \"nc\", \"ilp\": 8, \"us\": %.2f, "
                   "\"Ggather_s\": %.1f}\n", ncols, cf.threads, cf.bps, t[0][1] * 1e3, n / (t[0][1] * 1e-3) / 1e9);
            printf("{\"ncols\": %ld, \"threads\": %d, \"blocks_per_sm\": %d, \"flavor\": \"nc\", \"ilp\": 16, \"us\": %.2f, "
                   "\"Ggather_s\": %.1f}\n", ncols, cf.threads, cf.bps, t[0][2] * 1e3, n / (t[0][2] * 1e-3) / 1e9);
        }
    }
    return 0;
}
