#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#define CK(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char *s; cuGetErrorString(r, &s); printf("%s -> %d %s\n", #x, (int)r, s); return 1; } } while (0)
__global__ void red(unsigned long long *mc, unsigned long long v) {
    asm volatile("multimem.red.relaxed.sys.global.min.u64 [%0], %1;" :: "l"(mc + threadIdx.x), "l"(v + threadIdx.x) : "memory");
}
int main() {
    cudaFree(0);
    CUdevice dev; CK(cuDeviceGet(&dev, 0));
    int mcs = 0; CK(cuDeviceGetAttribute(&mcs, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    printf("multicast supported: %d\n", mcs);
    if (!mcs) return 0;
    CUmulticastObjectProp prop = {};
    prop.numDevices = 1; prop.size = 2 << 20; prop.handleTypes = 0;
    size_t gran = 0; CK(cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    prop.size = ((prop.size + gran - 1) / gran) * gran;
    printf("granularity %zu size %zu\n", gran, prop.size);
    CUmemGenericAllocationHandle mh;
    const unsigned long long types[3] = {0, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_FABRIC};
    CUresult cr = CUDA_ERROR_INVALID_VALUE;
    for (int t = 0; t < 3 && cr != CUDA_SUCCESS; ++t) {
        prop.handleTypes = types[t];
        cr = cuMulticastCreate(&mh, &prop);
        const char *es; cuGetErrorString(cr, &es);
        printf("cuMulticastCreate handleTypes=%llu -> %d %s\n", types[t], (int)cr, es);
    }
    if (cr != CUDA_SUCCESS) return 1;
    CK(cuMulticastAddDevice(mh, dev));
    CUmemAllocationProp ap = {}; ap.type = CU_MEM_ALLOCATION_TYPE_PINNED; ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ap.location.id = 0; ap.requestedHandleTypes = (CUmemAllocationHandleType)prop.handleTypes;
    CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, prop.size, &ap, 0));
    CK(cuMulticastBindMem(mh, 0, ph, 0, prop.size, 0));
    CUdeviceptr uc, mcp;
    CK(cuMemAddressReserve(&uc, prop.size, gran, 0, 0)); CK(cuMemMap(uc, prop.size, 0, ph, 0));
    CUmemAccessDesc ad = {}; ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad.location.id = 0; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, prop.size, &ad, 1));
    CK(cuMemAddressReserve(&mcp, prop.size, gran, 0, 0)); CK(cuMemMap(mcp, prop.size, 0, mh, 0)); CK(cuMemSetAccess(mcp, prop.size, &ad, 1));
    cudaMemset((void *)uc, 0xFF, 256 * 8);
    red<<<1, 256>>>((unsigned long long *)mcp, 1000);
    red<<<1, 256>>>((unsigned long long *)mcp, 500);
    cudaError_t e = cudaDeviceSynchronize(); printf("kernel: %s\n", cudaGetErrorString(e));
    unsigned long long h[4]; cudaMemcpy(h, (void *)uc, 32, cudaMemcpyDeviceToHost);
    printf("values %llu %llu %llu %llu (expect 500 501 502 503)\n", h[0], h[1], h[2], h[3]);
    return 0;
}
