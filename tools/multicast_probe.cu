// Probe (NEXT-2 feasibility): can this box create an NVLink multicast object on
// one device, bind device memory to it, and store through it with multimem.st?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o build/multicast_probe tools/multicast_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>

#define CK(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char *s = nullptr; cuGetErrorString(r, &s); \
    printf("%s -> %d (%s)\n", #x, (int)r, s ? s : "?"); return 1; } } while (0)

__global__ void k_mc_store(uint32_t *mc, int n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (4 * i + 3 < n) {
        uint32_t *a = mc + 4 * i;
        asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(a), "r"(4 * i), "r"(4 * i + 1),
                     "r"(4 * i + 2), "r"(4 * i + 3)
                     : "memory");
    }
}

int main() {
    CK(cuInit(0));
    CUdevice dev;
    CK(cuDeviceGet(&dev, 0));
    int mc = -1, fab = -1, ndev = 0;
    cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
    cudaGetDeviceCount(&ndev);
    printf("devices visible %d, MULTICAST_SUPPORTED %d\n", ndev, mc);
    cuDeviceGetAttribute(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev);
    printf("HANDLE_TYPE_FABRIC_SUPPORTED %d\n", fab);
    CUcontext ctx;
    CK(cuDevicePrimaryCtxRetain(&ctx, dev));
    CK(cuCtxSetCurrent(ctx));
    CUmulticastObjectProp p = {};
    p.numDevices = 1;
    const char *ht = getenv("MC_HANDLE");  // none | fd | fabric
    const CUmemAllocationHandleType hty = !ht ? CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR
                                         : (ht[0] == 'n' ? CU_MEM_HANDLE_TYPE_NONE
                                            : ht[0] == 'f' && ht[1] == 'a' ? CU_MEM_HANDLE_TYPE_FABRIC
                                                                           : CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
    p.handleTypes = hty;
    printf("handle type %d\n", (int)hty);
    size_t gran = 0;
    p.size = 2 << 20;
    CK(cuMulticastGetGranularity(&gran, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    p.size = (p.size + gran - 1) / gran * gran;
    printf("multicast granularity %zu, size %zu\n", gran, p.size);
    CUmemGenericAllocationHandle mch;
    CK(cuMulticastCreate(&mch, &p));
    CK(cuMulticastAddDevice(mch, dev));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = 0;
    ap.requestedHandleTypes = hty;
    CUmemGenericAllocationHandle mem;
    CK(cuMemCreate(&mem, p.size, &ap, 0));
    CK(cuMulticastBindMem(mch, 0, mem, 0, p.size, 0));
    CUdeviceptr uc, mcp;
    CK(cuMemAddressReserve(&uc, p.size, gran, 0, 0));
    CK(cuMemMap(uc, p.size, 0, mem, 0));
    CK(cuMemAddressReserve(&mcp, p.size, gran, 0, 0));
    CK(cuMemMap(mcp, p.size, 0, mch, 0));
    CUmemAccessDesc ad = {};
    ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ad.location.id = 0;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, p.size, &ad, 1));
    CK(cuMemSetAccess(mcp, p.size, &ad, 1));
    const int n = 1 << 16;
    cudaMemset((void *)uc, 0, n * 4);
    k_mc_store<<<n / 4 / 256, 256>>>((uint32_t *)mcp, n);
    cudaError_t e = cudaDeviceSynchronize();
    printf("multimem.st kernel: %s\n", cudaGetErrorString(e));
    static uint32_t h[1 << 16];
    cudaMemcpy(h, (void *)uc, n * 4, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < n; ++i) bad += h[i] != (uint32_t)i;
    printf("read back through the unicast mapping: %d of %d words wrong\n", bad, n);
    return bad != 0;
}
