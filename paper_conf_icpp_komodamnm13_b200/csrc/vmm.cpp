// Driver-API VMM and NVLS multicast helpers (vmm.h).
#include "vmm.h"

#include <cuda.h>
#include <cuda_runtime_api.h>
#include <unistd.h>

namespace accmg {
namespace vmm {
namespace {

struct Api {
    CUresult (*MemCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long);
    CUresult (*MemRelease)(CUmemGenericAllocationHandle);
    CUresult (*MemAddressReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
    CUresult (*MemAddressFree)(CUdeviceptr, size_t);
    CUresult (*MemMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
    CUresult (*MemUnmap)(CUdeviceptr, size_t);
    CUresult (*MemSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
    CUresult (*MemGetAllocationGranularity)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags);
    CUresult (*MemExportToShareableHandle)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType,
                                           unsigned long long);
    CUresult (*MemImportFromShareableHandle)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType);
    CUresult (*MulticastCreate)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*);
    CUresult (*MulticastAddDevice)(CUmemGenericAllocationHandle, CUdevice);
    CUresult (*MulticastBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                                 unsigned long long);
    CUresult (*MulticastUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
    CUresult (*MulticastGetGranularity)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags);
    CUresult (*DeviceGet)(CUdevice*, int);
    CUresult (*GetErrorString)(CUresult, const char**);
    bool ok = false;
    std::string missing;
};

template <typename F>
bool load(const char* name, F* fn, std::string* missing) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess ||
        !p) {
        if (missing->empty()) *missing = name;
        return false;
    }
    *fn = reinterpret_cast<F>(p);
    return true;
}

Api& api() {
    static Api a = [] {
        Api x{};
        std::string m;
        bool ok = load("cuMemCreate", &x.MemCreate, &m);
        ok &= load("cuMemRelease", &x.MemRelease, &m);
        ok &= load("cuMemAddressReserve", &x.MemAddressReserve, &m);
        ok &= load("cuMemAddressFree", &x.MemAddressFree, &m);
        ok &= load("cuMemMap", &x.MemMap, &m);
        ok &= load("cuMemUnmap", &x.MemUnmap, &m);
        ok &= load("cuMemSetAccess", &x.MemSetAccess, &m);
        ok &= load("cuMemGetAllocationGranularity", &x.MemGetAllocationGranularity, &m);
        ok &= load("cuMemExportToShareableHandle", &x.MemExportToShareableHandle, &m);
        ok &= load("cuMemImportFromShareableHandle", &x.MemImportFromShareableHandle, &m);
        ok &= load("cuMulticastCreate", &x.MulticastCreate, &m);
        ok &= load("cuMulticastAddDevice", &x.MulticastAddDevice, &m);
        ok &= load("cuMulticastBindMem", &x.MulticastBindMem, &m);
        ok &= load("cuMulticastUnbind", &x.MulticastUnbind, &m);
        ok &= load("cuMulticastGetGranularity", &x.MulticastGetGranularity, &m);
        ok &= load("cuDeviceGet", &x.DeviceGet, &m);
        ok &= load("cuGetErrorString", &x.GetErrorString, &m);
        x.ok = ok;
        x.missing = m;
        return x;
    }();
    return a;
}

bool check(CUresult r, const char* what, std::string* err) {
    if (r == CUDA_SUCCESS) return true;
    const char* s = "unknown";
    if (api().GetErrorString) api().GetErrorString(r, &s);
    if (err) *err = std::string(what) + ": " + s;
    return false;
}

CUmemAllocationProp phys_prop(int device) {
    CUmemAllocationProp p{};
    p.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    p.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    p.location.id = device;
    p.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    return p;
}

CUmulticastObjectProp mc_prop(int ndev, size_t bytes) {
    CUmulticastObjectProp p{};
    p.numDevices = (unsigned)ndev;
    p.size = bytes;
    p.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    return p;
}

// reserve a VA range for `h`, map it and give `device` read-write access
int map_rw(int device, CUmemGenericAllocationHandle h, size_t bytes, void** out, std::string* err) {
    Api& A = api();
    CUdeviceptr va = 0;
    if (!check(A.MemAddressReserve(&va, bytes, 0, 0, 0), "cuMemAddressReserve", err)) return -1;
    if (!check(A.MemMap(va, bytes, 0, h, 0), "cuMemMap", err)) {
        A.MemAddressFree(va, bytes);
        return -1;
    }
    CUmemAccessDesc ad{};
    ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ad.location.id = device;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (!check(A.MemSetAccess(va, bytes, &ad, 1), "cuMemSetAccess", err)) {
        A.MemUnmap(va, bytes);
        A.MemAddressFree(va, bytes);
        return -1;
    }
    *out = reinterpret_cast<void*>(va);
    return 0;
}

void unmap(void* ptr, size_t bytes) {
    if (!ptr) return;
    api().MemUnmap(reinterpret_cast<CUdeviceptr>(ptr), bytes);
    api().MemAddressFree(reinterpret_cast<CUdeviceptr>(ptr), bytes);
}

}  // namespace

bool available(std::string* why) {
    if (!api().ok && why) *why = "driver entry point missing: " + api().missing;
    return api().ok;
}

size_t round_up(int device, size_t bytes, bool multicast) {
    size_t g = 2u << 20;
    const CUmemAllocationProp pp = phys_prop(device);
    size_t pg = 0;
    if (api().MemGetAllocationGranularity(&pg, &pp, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) == CUDA_SUCCESS && pg > g)
        g = pg;
    if (multicast) {
        const CUmulticastObjectProp mp = mc_prop(1, bytes);
        size_t mg = 0;
        if (api().MulticastGetGranularity(&mg, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) == CUDA_SUCCESS && mg > g)
            g = mg;
    }
    return (bytes + g - 1) / g * g;
}

int alloc(int device, size_t bytes, Phys* out, std::string* err) {
    const CUmemAllocationProp pp = phys_prop(device);
    CUmemGenericAllocationHandle h = 0;
    if (!check(api().MemCreate(&h, bytes, &pp, 0), "cuMemCreate", err)) return -1;
    void* p = nullptr;
    if (map_rw(device, h, bytes, &p, err) != 0) {
        api().MemRelease(h);
        return -1;
    }
    out->handle = h;
    out->ptr = p;
    out->bytes = bytes;
    return 0;
}

int export_fd(const Phys& p, int* fd, std::string* err) {
    int f = -1;
    if (!check(api().MemExportToShareableHandle(&f, p.handle, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0),
               "cuMemExportToShareableHandle", err))
        return -1;
    *fd = f;
    return 0;
}

int import_map(int device, int fd, size_t bytes, Map* out, std::string* err) {
    CUmemGenericAllocationHandle h = 0;
    const bool ok = check(api().MemImportFromShareableHandle(&h, reinterpret_cast<void*>((uintptr_t)fd),
                                                             CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR),
                          "cuMemImportFromShareableHandle", err);
    ::close(fd);
    if (!ok) return -1;
    void* p = nullptr;
    if (map_rw(device, h, bytes, &p, err) != 0) {
        api().MemRelease(h);
        return -1;
    }
    out->handle = h;
    out->ptr = p;
    out->bytes = bytes;
    return 0;
}

void release(Phys* p) {
    if (!p->handle) return;
    unmap(p->ptr, p->bytes);
    api().MemRelease(p->handle);
    *p = Phys{};
}

void release(Map* m) {
    if (!m->handle) return;
    unmap(m->ptr, m->bytes);
    api().MemRelease(m->handle);
    *m = Map{};
}

void unmap_only(Map* m) {
    unmap(m->ptr, m->bytes);
    *m = Map{};
}

int mc_probe(int ndev, size_t bytes, std::string* why) {
    if (!available(why)) return -1;
    const CUmulticastObjectProp mp = mc_prop(ndev, bytes);
    size_t g = 0;
    if (!check(api().MulticastGetGranularity(&g, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED),
               "cuMulticastGetGranularity", why))
        return -1;
    CUmulticastObjectProp p2 = mp;
    p2.size = (bytes + g - 1) / g * g;
    CUmemGenericAllocationHandle mc = 0;
    if (!check(api().MulticastCreate(&mc, &p2), "cuMulticastCreate", why)) return -1;
    api().MemRelease(mc);
    return 0;
}

int mc_create(int ndev, size_t bytes, unsigned long long* mc, std::string* err) {
    const CUmulticastObjectProp mp = mc_prop(ndev, bytes);
    CUmemGenericAllocationHandle h = 0;
    if (!check(api().MulticastCreate(&h, &mp), "cuMulticastCreate", err)) return -1;
    *mc = h;
    return 0;
}

int mc_export_fd(unsigned long long mc, int* fd, std::string* err) {
    int f = -1;
    if (!check(api().MemExportToShareableHandle(&f, mc, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0),
               "cuMemExportToShareableHandle(multicast)", err))
        return -1;
    *fd = f;
    return 0;
}

int mc_import(int fd, unsigned long long* mc, std::string* err) {
    CUmemGenericAllocationHandle h = 0;
    const bool ok = check(api().MemImportFromShareableHandle(&h, reinterpret_cast<void*>((uintptr_t)fd),
                                                             CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR),
                          "cuMemImportFromShareableHandle(multicast)", err);
    ::close(fd);
    if (!ok) return -1;
    *mc = h;
    return 0;
}

int mc_add_device(unsigned long long mc, int device, std::string* err) {
    CUdevice d = 0;
    if (!check(api().DeviceGet(&d, device), "cuDeviceGet", err)) return -1;
    return check(api().MulticastAddDevice(mc, d), "cuMulticastAddDevice", err) ? 0 : -1;
}

int mc_bind(unsigned long long mc, const Phys& p, std::string* err) {
    return check(api().MulticastBindMem(mc, 0, p.handle, 0, p.bytes, 0), "cuMulticastBindMem", err) ? 0 : -1;
}

int mc_map(int device, unsigned long long mc, size_t bytes, Map* out, std::string* err) {
    void* p = nullptr;
    if (map_rw(device, mc, bytes, &p, err) != 0) return -1;
    out->handle = 0;  // the object is released by mc_release, not by the mapping
    out->ptr = p;
    out->bytes = bytes;
    return 0;
}

void mc_release(unsigned long long mc, int device, size_t bytes, bool bound) {
    if (!mc) return;
    CUdevice d = 0;
    if (bound && api().DeviceGet(&d, device) == CUDA_SUCCESS) api().MulticastUnbind(mc, d, 0, bytes);
    api().MemRelease(mc);
}

}  // namespace vmm
}  // namespace accmg
