// tools/mcbuf.cu -- test / measurement helper (not the method): an NVLink-SHARP (NVLS) multicast buffer on the
// GPUs of this process, built with the CUDA driver's multicast objects (cuMulticastCreate / cuMulticastBindMem).
// A multicast address (mc) addresses one allocation on every member GPU: one multimem.st from a kernel lands in
// all of them through the NVSwitch.  On a multi-GPU node the product path gets these addresses from torch
// symmetric memory (ShardedSpMM.symmetric_C: multicast_ptr); this helper makes the same store path testable on
// ONE GPU (a one-member multicast object: the store reaches the local allocation, read back through its unicast
// address uc).
//   mcbuf_create(bytes, &uc, &mc, &handle) -> 0 ok, else a CUresult / -1 (multicast unsupported)
//   mcbuf_destroy(handle)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

struct McBuf {
    CUmemGenericAllocationHandle mem = 0;
    CUmemGenericAllocationHandle mch = 0;
    CUdeviceptr uc = 0, mc = 0;
    size_t size = 0;
    CUdevice dev = 0;
};

static int g_mc_fail_line = 0;   // source line of the first failing driver call (diagnostics)
#define MC_TRY(x)                                                  \
    do {                                                           \
        CUresult r_ = (x);                                         \
        if (r_ != CUDA_SUCCESS) { g_mc_fail_line = __LINE__; return (int)r_; } \
    } while (0)
extern "C" int mcbuf_fail_line(void) { return g_mc_fail_line; }

static int mcbuf_create_ht(size_t bytes, void **uc, void **mc, void **handle, CUmemAllocationHandleType ht);
// POSIX file-descriptor handles (HGX NVSwitch nodes), else fabric handles (IMEX / multi-node NVLink domains)
extern "C" int mcbuf_create(size_t bytes, void **uc, void **mc, void **handle) {
    const int rc = mcbuf_create_ht(bytes, uc, mc, handle, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
    if (rc == 0 || rc == -1) return rc;
    const int line = g_mc_fail_line;
    const int rc2 = mcbuf_create_ht(bytes, uc, mc, handle, CU_MEM_HANDLE_TYPE_FABRIC);
    if (rc2 != 0) g_mc_fail_line = line * 1000 + g_mc_fail_line;   // both attempts' failing lines
    return rc2;
}

static int mcbuf_create_ht(size_t bytes, void **uc, void **mc, void **handle, CUmemAllocationHandleType ht) {
    cudaFree(0);   // primary context
    int d = 0;
    cudaGetDevice(&d);
    McBuf *b = new McBuf();
    MC_TRY(cuDeviceGet(&b->dev, d));
    int supported = 0;
    MC_TRY(cuDeviceGetAttribute(&supported, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, b->dev));
    if (!supported) { delete b; return -1; }
    CUmulticastObjectProp prop = {};
    prop.numDevices = 1;
    prop.handleTypes = ht;
    prop.size = bytes;
    size_t gran = 0, agran = 0;
    MC_TRY(cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_MINIMUM));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = b->dev;
    ap.requestedHandleTypes = ht;
    MC_TRY(cuMemGetAllocationGranularity(&agran, &ap, CU_MEM_ALLOC_GRANULARITY_MINIMUM));
    const size_t g = gran > agran ? gran : agran;   // both are powers of two: the larger is a multiple of both
    b->size = (bytes + g - 1) / g * g;
    prop.size = b->size;
    MC_TRY(cuMulticastCreate(&b->mch, &prop));
    MC_TRY(cuMulticastAddDevice(b->mch, b->dev));
    MC_TRY(cuMemCreate(&b->mem, b->size, &ap, 0));
    MC_TRY(cuMulticastBindMem(b->mch, 0, b->mem, 0, b->size, 0));
    CUmemAccessDesc acc = {};
    acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc.location.id = b->dev;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    MC_TRY(cuMemAddressReserve(&b->uc, b->size, g, 0, 0));
    MC_TRY(cuMemMap(b->uc, b->size, 0, b->mem, 0));
    MC_TRY(cuMemSetAccess(b->uc, b->size, &acc, 1));
    MC_TRY(cuMemAddressReserve(&b->mc, b->size, g, 0, 0));
    MC_TRY(cuMemMap(b->mc, b->size, 0, b->mch, 0));
    MC_TRY(cuMemSetAccess(b->mc, b->size, &acc, 1));
    *uc = (void *)b->uc;
    *mc = (void *)b->mc;
    *handle = b;
    return 0;
}

extern "C" void mcbuf_destroy(void *handle) {
    McBuf *b = (McBuf *)handle;
    if (!b) return;
    cudaDeviceSynchronize();
    if (b->mc) { cuMemUnmap(b->mc, b->size); cuMemAddressFree(b->mc, b->size); }
    if (b->uc) { cuMemUnmap(b->uc, b->size); cuMemAddressFree(b->uc, b->size); }
    if (b->mch) { cuMulticastUnbind(b->mch, b->dev, 0, b->size); cuMemRelease(b->mch); }
    if (b->mem) cuMemRelease(b->mem);
    delete b;
}

#ifdef MCBUF_MAIN
__global__ void k_st(float4 *mc, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const float v = (float)i;
        asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(mc + i), "f"(v), "f"(v + 1.f),
                     "f"(v + 2.f), "f"(v + 3.f) : "memory");
    }
}
int main() {
    void *uc, *mc, *h;
    const int64_t n = 1 << 20;
    int rc = mcbuf_create(n * 16, &uc, &mc, &h);
    printf("mcbuf_create rc=%d line=%d\n", rc, mcbuf_fail_line());
    {
        CUdevice dv; cuDeviceGet(&dv, 0); int a1 = 0, a2 = 0, a3 = 0;
        cuDeviceGetAttribute(&a1, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dv);
        cuDeviceGetAttribute(&a2, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dv);
        cuDeviceGetAttribute(&a3, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR_SUPPORTED, dv);
        printf("multicast_supported=%d fabric=%d posix_fd=%d\n", a1, a2, a3);
    }
    if (rc) return 1;
    k_st<<<148, 256>>>((float4 *)mc, n);
    cudaError_t e = cudaDeviceSynchronize();
    float4 x;
    cudaMemcpy(&x, (float4 *)uc + 12345, 16, cudaMemcpyDeviceToHost);
    printf("kernel %s; uc[12345] = %g %g %g %g\n", cudaGetErrorString(e), x.x, x.y, x.z, x.w);
    mcbuf_destroy(h);
    return 0;
}
#endif
