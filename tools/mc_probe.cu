// probe: is NVLS multicast usable on this box (1 GPU)?  cuMulticastCreate with one device,
// bind 2 MB, map the multicast handle, multimem.st from a kernel, read back via the unicast VA.
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>
#define CKD(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char *s; cuGetErrorString(r, &s); printf("FAIL %s: %s\n", #x, s); return 1; } } while (0)
__global__ void st_mc(double *mc, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) { double v = i * 0.5; asm volatile("multimem.st.global.f64 [%0], %1;" :: "l"(mc + i), "d"(v) : "memory"); }
}
int main() {
    CKD(cuInit(0));
    CUdevice dev; CKD(cuDeviceGet(&dev, 0));
    CUcontext ctx; CKD(cuDevicePrimaryCtxRetain(&ctx, dev)); CKD(cuCtxSetCurrent(ctx));
    int mc = -1; CKD(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    printf("multicast supported: %d\n", mc);
    if (!mc) return 0;
    CUmulticastObjectProp prop = {};
    CUmemGenericAllocationHandle mch;
    int created = 0;
    const int nds[] = {1, 2};
    const unsigned long long hts[] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_NONE, CU_MEM_HANDLE_TYPE_FABRIC};
    for (int a = 0; a < 2 && !created; a++)
        for (int b = 0; b < 3 && !created; b++) {
            prop = {};
            prop.numDevices = nds[a]; prop.handleTypes = hts[b]; prop.size = 2 << 20;
            size_t gran = 0;
            if (cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS) continue;
            prop.size = ((prop.size + gran - 1) / gran) * gran;
            CUresult r = cuMulticastCreate(&mch, &prop);
            const char *es; cuGetErrorString(r, &es);
            printf("cuMulticastCreate numDevices=%d handleTypes=%llu: %s\n", nds[a], hts[b], es);
            if (r == CUDA_SUCCESS) created = 1;
        }
    if (!created) return 0;
    if (prop.numDevices > 1) { printf("only a >= 2-device multicast object is creatable; cannot complete it on 1 GPU\n"); return 0; }
    CKD(cuMulticastAddDevice(mch, dev));
    CUmemAllocationProp ap = {}; ap.type = CU_MEM_ALLOCATION_TYPE_PINNED; ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ap.location.id = dev;
    ap.requestedHandleTypes = (CUmemAllocationHandleType)prop.handleTypes;
    CUmemGenericAllocationHandle mh; CKD(cuMemCreate(&mh, prop.size, &ap, 0));
    CKD(cuMulticastBindMem(mch, 0, mh, 0, prop.size, 0));
    CUdeviceptr uva, mva;
    CKD(cuMemAddressReserve(&uva, prop.size, 0, 0, 0)); CKD(cuMemMap(uva, prop.size, 0, mh, 0));
    CKD(cuMemAddressReserve(&mva, prop.size, 0, 0, 0)); CKD(cuMemMap(mva, prop.size, 0, mch, 0));
    CUmemAccessDesc ad = {}; ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad.location.id = dev; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CKD(cuMemSetAccess(uva, prop.size, &ad, 1)); CKD(cuMemSetAccess(mva, prop.size, &ad, 1));
    const int n = 1000;
    st_mc<<<4, 256>>>((double *)mva, n);
    cudaError_t e = cudaDeviceSynchronize(); printf("kernel: %s\n", cudaGetErrorString(e));
    double h[n]; cudaMemcpy(h, (void *)uva, sizeof(h), cudaMemcpyDeviceToHost);
    int ok = 1; for (int i = 0; i < n; i++) ok &= h[i] == i * 0.5;
    printf("multimem.st readback %s\n", ok ? "OK" : "MISMATCH");
    return 0;
}
