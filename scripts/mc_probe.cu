// Probe: NVLS multicast on one B200 — create a multicast object, bind a physical allocation, map
// the multicast address and write through it with multimem.st; read back via the unicast mapping.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#define CK(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char* s; cuGetErrorString(r, &s); printf("%s -> %s\n", #x, s); return 1; } } while (0)

__global__ void mc_store(float* mc, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" ::"l"(mc + i), "f"(1.5f * i) : "memory");
}

int try_type(CUmemAllocationHandleType ht, const char* name) {
    CUdevice dev; CK(cuDeviceGet(&dev, 0));
    CUmulticastObjectProp mp = {};
    mp.numDevices = 1; mp.handleTypes = ht; mp.size = 2 << 20;
    size_t g = 0;
    CK(cuMulticastGetGranularity(&g, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    mp.size = g;
    CUmemGenericAllocationHandle mc;
    CUresult r = cuMulticastCreate(&mc, &mp);
    if (r != CUDA_SUCCESS) { const char* s; cuGetErrorString(r, &s); printf("[%s] create: %s\n", name, s); return 1; }
    CK(cuMulticastAddDevice(mc, dev));
    CUmemAllocationProp pp = {};
    pp.type = CU_MEM_ALLOCATION_TYPE_PINNED; pp.location.type = CU_MEM_LOCATION_TYPE_DEVICE; pp.location.id = 0;
    pp.requestedHandleTypes = ht;
    size_t pg = 0; CK(cuMemGetAllocationGranularity(&pg, &pp, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
    CUmemGenericAllocationHandle ph; CK(cuMemCreate(&ph, mp.size, &pp, 0));
    CK(cuMulticastBindMem(mc, 0, ph, 0, mp.size, 0));
    CUdeviceptr uc, mcp;
    CK(cuMemAddressReserve(&uc, mp.size, g, 0, 0)); CK(cuMemMap(uc, mp.size, 0, ph, 0));
    CK(cuMemAddressReserve(&mcp, mp.size, g, 0, 0)); CK(cuMemMap(mcp, mp.size, 0, mc, 0));
    CUmemAccessDesc ad = {}; ad.location = pp.location; ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, mp.size, &ad, 1)); CK(cuMemSetAccess(mcp, mp.size, &ad, 1));
    int n = 1 << 16;
    cudaMemset((void*)uc, 0, n * 4);
    mc_store<<<n / 256, 256>>>((float*)mcp, n);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<float> h(n);
    cudaMemcpy(h.data(), (void*)uc, n * 4, cudaMemcpyDeviceToHost);
    int bad = 0; for (int i = 0; i < n; ++i) bad += h[i] != 1.5f * i;
    printf("[%s] multicast gran %zu, kernel %s, mismatches %d\n", name, g, cudaGetErrorString(e), bad);
    return 0;
}

int main() {
    CK(cuInit(0)); cudaFree(0);
    try_type(CU_MEM_HANDLE_TYPE_NONE, "none");
    try_type(CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, "posix_fd");
    try_type(CU_MEM_HANDLE_TYPE_FABRIC, "fabric");
    return 0;
}
