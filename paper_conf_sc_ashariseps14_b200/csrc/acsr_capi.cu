// acsr_capi.cu -- status strings, thread-local error text, device queries.
#include <mutex>
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>

#include "acsr_internal.cuh"

static thread_local char g_err[512] = "";

void acsr_set_error(const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

acsr_status acsr_check_launch(const char *what)
{
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        acsr_set_error("%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
        return ACSR_ERR_CUDA;
    }
    return ACSR_OK;
}

bool acsr::acsr_pdl_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("ACSR_PDL");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}

// ACSR_CARVEOUT=<percent> (A/B knob, default unset): the preferred shared-memory carveout
// given to every kernel launched through launch_pdl, so consecutive kernels of a call
// chain (binning -> SpMV) can share one L1/shared split instead of the SM reconfiguring
// between them.
int acsr::acsr_carveout()
{
    static int v = -2;
    if (v == -2) {
        const char *e = getenv("ACSR_CARVEOUT");
        v = (e && e[0]) ? atoi(e) : -1;
        if (v > 100) v = 100;
    }
    return v;
}

bool acsr::acsr_carveout_once(const void *fn)
{
    static std::mutex mu;  // ctypes releases the GIL: launches can come from several host threads
    static const void *seen[128];
    static int n = 0;
    std::lock_guard<std::mutex> lock(mu);
    for (int i = 0; i < n; i++)
        if (seen[i] == fn) return false;
    if (n < 128) seen[n++] = fn;
    return true;
}

int acsr_num_sms()
{
    static int sms[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (!sms[dev]) {
        int v = 0;
        cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
        sms[dev] = v > 0 ? v : 148;
    }
    return sms[dev];
}

extern "C" const char *acsr_status_string(acsr_status s)
{
    switch (s) {
        case ACSR_OK: return "ACSR_OK";
        case ACSR_ERR_INVALID_VALUE: return "ACSR_ERR_INVALID_VALUE";
        case ACSR_ERR_WORKSPACE: return "ACSR_ERR_WORKSPACE";
        case ACSR_ERR_CAPACITY: return "ACSR_ERR_CAPACITY";
        case ACSR_ERR_CUDA: return "ACSR_ERR_CUDA";
        case ACSR_ERR_NCCL: return "ACSR_ERR_NCCL";
        case ACSR_ERR_UNSUPPORTED: return "ACSR_ERR_UNSUPPORTED";
    }
    return "ACSR_UNKNOWN_STATUS";
}

extern "C" const char *acsr_last_error(void) { return g_err; }

extern "C" int acsr_version(void) { return 100; }
