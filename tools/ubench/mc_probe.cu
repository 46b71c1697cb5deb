// NVLS multicast probe (one GPU): is a multicast object creatable here, and do
// multimem.red.or / multimem.ld_reduce.or on its address reach the bound memory?
// nvcc -gencode arch=compute_100a,code=sm_100a -o mc_probe mc_probe.cu -lcuda
#include <cuda.h>
#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char *s = nullptr; cuGetErrorString(r_, &s); \
    printf("FAIL %s -> %d %s\n", #x, (int)r_, s ? s : "?"); return 1; } } while (0)

__global__ void red_or(uint32_t *mc, int n)
{
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        asm volatile("multimem.red.relaxed.sys.global.or.b32 [%0], %1;" ::"l"(mc + i), "r"(1u << (i & 31)) : "memory");
}

__global__ void ld_or(const uint32_t *mc, uint32_t *out, int n)
{
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        uint32_t v;
        asm volatile("multimem.ld_reduce.relaxed.sys.global.or.b32 %0, [%1];" : "=r"(v) : "l"(mc + i) : "memory");
        out[i] = v;
    }
}

int main()
{
    CK(cuInit(0));
    CUdevice dev;
    CK(cuDeviceGet(&dev, 0));
    int mcs = -1;
    CK(cuDeviceGetAttribute(&mcs, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    printf("multicast_supported=%d\n", mcs);
    CUcontext ctx;
    CK(cuDevicePrimaryCtxRetain(&ctx, dev));
    CK(cuCtxSetCurrent(ctx));
    if (!mcs) return 0;
    CUmulticastObjectProp mp = {};
    mp.numDevices = 1;
    size_t gran = 0;
    mp.size = 1 << 21;
    CUmemGenericAllocationHandle mch;
    bool made = false;
    const CUmemAllocationHandleType types[] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_FABRIC,
                                               CU_MEM_HANDLE_TYPE_NONE};
    size_t size = 0;
    for (auto t : types) {
        mp.handleTypes = t;
        mp.size = 1 << 21;
        CUresult r = cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
        if (r != CUDA_SUCCESS) { printf("granularity(type %d) -> %d\n", (int)t, (int)r); continue; }
        size = ((size_t)(1 << 21) + gran - 1) / gran * gran;
        mp.size = size;
        r = cuMulticastCreate(&mch, &mp);
        printf("cuMulticastCreate(type %d, numDevices 1, size %zu, gran %zu) -> %d\n", (int)t, size, gran, (int)r);
        if (r == CUDA_SUCCESS) { made = true; break; }
    }
    if (!made) return 0;
    CK(cuMulticastAddDevice(mch, dev));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = dev;
    CUmemGenericAllocationHandle mem;
    CK(cuMemCreate(&mem, size, &ap, 0));
    CK(cuMulticastBindMem(mch, 0, mem, 0, size, 0));
    CUdeviceptr uc, mc;
    CK(cuMemAddressReserve(&uc, size, gran, 0, 0));
    CK(cuMemMap(uc, size, 0, mem, 0));
    CK(cuMemAddressReserve(&mc, size, gran, 0, 0));
    CK(cuMemMap(mc, size, 0, mch, 0));
    CUmemAccessDesc ad = {};
    ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ad.location.id = dev;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, size, &ad, 1));
    CK(cuMemSetAccess(mc, size, &ad, 1));
    const int n = 1 << 16;
    CK(cuMemsetD32(uc, 0x100, n));
    red_or<<<64, 256>>>(reinterpret_cast<uint32_t *>(mc), n);
    CK(cuCtxSynchronize());
    std::vector<uint32_t> h(n);
    CK(cuMemcpyDtoH(h.data(), uc, n * 4));
    int bad = 0;
    for (int i = 0; i < n; ++i) bad += h[i] != (0x100u | (1u << (i & 31)));
    printf("multimem.red.or via multicast VA: %s (%d bad)\n", bad ? "WRONG" : "ok", bad);
    CUdeviceptr out;
    CK(cuMemAlloc(&out, n * 4));
    ld_or<<<64, 256>>>(reinterpret_cast<const uint32_t *>(mc), reinterpret_cast<uint32_t *>(out), n);
    CK(cuCtxSynchronize());
    CK(cuMemcpyDtoH(h.data(), out, n * 4));
    bad = 0;
    for (int i = 0; i < n; ++i) bad += h[i] != (0x100u | (1u << (i & 31)));
    printf("multimem.ld_reduce.or via multicast VA: %s (%d bad)\n", bad ? "WRONG" : "ok", bad);
    return 0;
}
