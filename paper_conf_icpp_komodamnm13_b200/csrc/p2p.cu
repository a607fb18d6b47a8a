// Device-side BSP barrier across processes (one per GPU): the global barrier that closes every
// parallel loop (L64 §III.A), without a host round trip. Each rank owns an array sig[W] in its HBM,
// mapped into every peer through CUDA IPC (NVLink / NVSwitch). At epoch e, thread q of rank r
// stores e into sig_q[r] with release semantics at system scope, then spins until sig_r[q] >= e
// (acquire). All of rank r's earlier stream work (bodies, pushes into peer replicas) is complete
// and visible before its arrival is published, so after the barrier every rank may read what any
// peer wrote in the loop.
#include "kernels.h"

namespace accmg {
namespace k {
namespace {

__global__ void barrier_k(const PtrList peers, uint64_t* my_sig, int rank, int W, uint64_t epoch) {
    const int q = threadIdx.x;
    if (q >= W) return;
    uint64_t* dst = static_cast<uint64_t*>(peers.p[q]) + rank;
    __threadfence_system();
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(dst), "l"(epoch) : "memory");
    uint64_t v = 0;
    do {
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(my_sig + q) : "memory");
    } while (v < epoch);
}

// One CTA row per range (blockIdx.y), 16-byte vectors when both ends are 16-byte aligned.
__global__ void __launch_bounds__(256) copy_batch_k(const CopyList c) {
    const int r = blockIdx.y;
    if (r >= c.n) return;
    const uint8_t* src = static_cast<const uint8_t*>(c.src[r]);
    uint8_t* dst = static_cast<uint8_t*>(c.dst[r]);
    const int64_t nb = c.bytes[r];
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
    if (((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15) == 0) {
        const int64_t nv = nb / 16;
        const int4* s4 = reinterpret_cast<const int4*>(src);
        int4* d4 = reinterpret_cast<int4*>(dst);
        for (int64_t i = tid; i < nv; i += nth) d4[i] = s4[i];
        for (int64_t i = nv * 16 + tid; i < nb; i += nth) dst[i] = src[i];
    } else if (((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 3) == 0) {
        const int64_t nv = nb / 4;
        const uint32_t* s4 = reinterpret_cast<const uint32_t*>(src);
        uint32_t* d4 = reinterpret_cast<uint32_t*>(dst);
        for (int64_t i = tid; i < nv; i += nth) d4[i] = s4[i];
        for (int64_t i = nv * 4 + tid; i < nb; i += nth) dst[i] = src[i];
    } else {
        for (int64_t i = tid; i < nb; i += nth) dst[i] = src[i];
    }
}

}  // namespace

cudaError_t copy_batch(const CopyList& c, cudaStream_t s, int64_t* launches) {
    if (c.n == 0) return cudaSuccess;
    int64_t mx = 0;
    for (int i = 0; i < c.n; ++i) mx = c.bytes[i] > mx ? c.bytes[i] : mx;
    int64_t bx = (mx / 16 + 255) / 256;
    if (bx > 256) bx = 256;
    if (bx < 1) bx = 1;
    copy_batch_k<<<dim3((unsigned)bx, (unsigned)c.n), 256, 0, s>>>(c);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t device_barrier(const PtrList& peer_sigs, uint64_t* my_sig, int rank, int W, uint64_t epoch,
                           cudaStream_t s, int64_t* launches) {
    barrier_k<<<1, 64, 0, s>>>(peer_sigs, my_sig, rank, W, epoch);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
