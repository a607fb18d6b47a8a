// Host helpers of the kernel launchers: cuTensorMapEncodeTiled via the runtime's driver entry point
// (no libcuda link), and per-process caches of everything a launch needs that does not change
// between loops (one device per process): tensor maps keyed by their full argument list, the SM
// count, and per kernel the dynamic shared-memory attribute (set once) and the resident CTAs per SM.
// A loop launch then costs the kernel launch itself, not ~10 us of attribute and occupancy queries.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime_api.h>

#include <cstring>

namespace accmg {

inline PFN_cuTensorMapEncodeTiled_v12000 tma_encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }
    return fn;
}

// cuTensorMapEncodeTiled with a small cache: a map is a pure function of its arguments, so a hit
// returns the identical descriptor (ping-pong Jacobi buffers, the same partition every loop).
inline bool tma_encode_tiled(CUtensorMap* out, CUtensorMapDataType dt, cuuint32_t rank, void* base,
                             const cuuint64_t* dims, const cuuint64_t* strides, const cuuint32_t* box,
                             const cuuint32_t* es, CUtensorMapInterleave il, CUtensorMapSwizzle sw,
                             CUtensorMapL2promotion l2, CUtensorMapFloatOOBfill oob) {
    struct Key {
        void* base;
        cuuint64_t dims[5], strides[4];
        cuuint32_t box[5], es[5];
        int dt, rank, il, sw, l2, oob;
    };
    struct Entry {
        Key key;
        CUtensorMap map;
    };
    constexpr int kEntries = 64;
    static Entry cache[kEntries];
    static int used = 0, next = 0;
    Key k;
    std::memset(&k, 0, sizeof(k));
    k.base = base;
    for (cuuint32_t i = 0; i < rank && i < 5; ++i) {
        k.dims[i] = dims[i];
        k.box[i] = box[i];
        k.es[i] = es[i];
        if (i + 1 < rank) k.strides[i] = strides[i];
    }
    k.dt = (int)dt;
    k.rank = (int)rank;
    k.il = (int)il;
    k.sw = (int)sw;
    k.l2 = (int)l2;
    k.oob = (int)oob;
    for (int i = 0; i < used; ++i)
        if (std::memcmp(&cache[i].key, &k, sizeof(Key)) == 0) {
            *out = cache[i].map;
            return true;
        }
    auto fn = tma_encode_fn();
    if (!fn || fn(out, dt, rank, base, dims, strides, box, es, il, sw, l2, oob) != CUDA_SUCCESS) return false;
    Entry& e = cache[next];
    e.key = k;
    e.map = *out;
    next = (next + 1) % kEntries;
    if (used < kEntries) ++used;
    return true;
}

inline int sm_count_cached() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

// First launch of (kernel, block size, dynamic smem): raise the kernel's dynamic shared-memory limit
// if it is below smem (the limit is per kernel, so it only ever grows: a smaller launch must not
// lower it under a larger cached one), optionally prefer all of L1 as shared memory, and query the
// resident CTAs per SM; later launches read the cached answer.
template <typename K>
cudaError_t kernel_prep(K kern, int threads, size_t smem, int* per_sm = nullptr, bool max_carveout = false) {
    struct Entry {
        const void* fn;
        int threads;
        size_t smem;
        int per_sm;
    };
    struct Limit {
        const void* fn;
        size_t smem;
    };
    constexpr int kEntries = 128;
    static Entry cache[kEntries];
    static Limit limits[kEntries];
    static int used = 0, nlim = 0;
    const void* f = reinterpret_cast<const void*>(kern);
    for (int i = 0; i < used; ++i)
        if (cache[i].fn == f && cache[i].threads == threads && cache[i].smem == smem) {
            if (per_sm) *per_sm = cache[i].per_sm;
            return cudaSuccess;
        }
    int li = 0;
    while (li < nlim && limits[li].fn != f) ++li;
    if (li == nlim || limits[li].smem < smem) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        if (max_carveout) {
            e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     cudaSharedmemCarveoutMaxShared);
            if (e != cudaSuccess) return e;
        }
        if (li == nlim && nlim < kEntries) limits[nlim++] = {f, smem};
        else if (li < nlim) limits[li].smem = smem;
    }
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, threads, smem) != cudaSuccess) {
        (void)cudaGetLastError();  // the launch itself reports real errors; assume one CTA per SM
        n = 1;
    }
    if (n < 1) n = 1;
    if (used < kEntries) cache[used++] = {f, threads, smem, n};
    if (per_sm) *per_sm = n;
    return cudaSuccess;
}

}  // namespace accmg
