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

}  // namespace

cudaError_t device_barrier(const PtrList& peer_sigs, uint64_t* my_sig, int rank, int W, uint64_t epoch,
                           cudaStream_t s, int64_t* launches) {
    barrier_k<<<1, 64, 0, s>>>(peer_sigs, my_sig, rank, W, epoch);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
