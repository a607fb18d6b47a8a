// accmg runtime: the C ABI of include/accmg.h.
//
// Host side of one offloaded parallel loop (§III.A, three BSP steps):
//   1. task mapping (L108): dim 0 of the iteration space is divided into P contiguous chunks;
//   2. data loader (L117-125 §IV.C): per region, each partition needs its declared window
//      (distribution policy, L121-123) or the whole array (replica policy, L121); what it does not
//      already hold is pulled — from the partition that holds it (device copy or NCCL) or from the
//      host copy — and nothing moves when the read pattern repeats (L125);
//   3. body kernels on every local partition (loop bodies of csrc/*.cu);
//   4. inter-GPU communication manager (L127-137 §IV.D): declared writes move ownership (the data
//      follows lazily when a later loop reads it); undeclared writes were tracked with two-level
//      dirty bits, are compacted into packed runs and scattered into every other replica;
//      reductiontoarray destinations are merged block -> GPU -> across GPUs (L112);
//   5. global barrier (L64): stream order on each process; NCCL ops order across processes.
//
// State per region: one full-extent replica per local partition (global indices, so the index
// rewriting of L110 is the identity) and a validity table: for every partition (all ranks keep the
// whole table, identical everywhere because every call is collective) the set of element intervals
// whose value there is current, plus this process's host-copy validity.
#include "accmg.h"

#include <cuda_runtime_api.h>
#include <fcntl.h>
#include <unistd.h>

#include <algorithm>
#include <map>
#include <unordered_map>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "bootstrap.h"
#include "intervals.h"
#include "kernels.h"
#include "nccl_dl.h"
#include "vmm.h"

#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges cost a pointer test unless a tool is attached

using accmg::IntervalSet;
using accmg::Ival;
namespace k = accmg::k;

namespace {

struct Trk {  // dirty-bit tracking + packed send buffer of one local replica (L133-135)
    uint32_t* l1 = nullptr;
    uint32_t* l2 = nullptr;
    int64_t nwords = 0, nl2 = 0, ntiles = 0;
    int64_t* tile_counts = nullptr;
    int64_t* tile_offs = nullptr;
    uint32_t* tile_edges = nullptr;
    int64_t* totals = nullptr;  // device {n_runs, n_elems, dirty_chunks, n_run_ends}
    uint8_t* packed = nullptr;
    int64_t packed_cap = 0, packed_bytes = 0, n_runs = 0, n_elems = 0, dirty_chunks = 0;
    uint32_t* snap_l1 = nullptr;
    uint32_t* snap_l2 = nullptr;
    bool has_snap = false, has_packed = false;
};

}  // namespace

struct accmg_region_s {
    int64_t id = 0;
    uint8_t* host = nullptr;
    int64_t esize = 0, extent = 0;
    // Local replicas: dev[li] is the *global-index base* of partition li's replica — element e lives
    // at dev[li] + e*esize — but only the hull of what the partition ever needs is allocated
    // (window-sized allocations for distributed arrays, §8 row f4; full extent for replicated ones).
    std::vector<uint8_t*> dev;       // V (virtual bases; nullptr = nothing allocated yet)
    std::vector<uint8_t*> abase;     // V cudaMalloc'd pointers
    std::vector<Ival> arange;        // P allocated element range of every partition (global table)
    std::vector<IntervalSet> valid;  // P partitions
    std::vector<IntervalSet> last_read;  // P: declared read windows of the last loop that read this
                                         // region (halo-push prediction, L125); empty = no prediction
    IntervalSet host_valid;          // this process's host copy
    std::vector<Trk> trk;            // V
    std::vector<int64_t*> partial;   // V reduction partials (REDUCE_SUM)
    // P2P mode (one process per GPU): this process's view of EVERY partition's replica / partial
    // (local allocations, or peer allocations mapped through CUDA IPC)
    std::vector<uint8_t*> gdev;      // P
    std::vector<int64_t*> gpartial;  // P
    int64_t* acc = nullptr;          // local reduction accumulator (P2P mode)
    std::vector<void*> opened;       // IPC mappings of the peers' replicas (re-opened when a hull grows)
    std::vector<void*> opened_partial;  // IPC mappings of the peers' reduction partials (opened once)
    // §8 row f3 (config.multicast, P2P mode): the replica is a driver-VMM allocation shared with the
    // peers through file descriptors (vpeer: their replicas mapped here), and, where the node can
    // create one, bound to an NVLS multicast object mapped at mcmap
    bool vmm = false;
    accmg::vmm::Phys vphys;
    std::vector<accmg::vmm::Map> vpeer;
    unsigned long long mc = 0;
    accmg::vmm::Map mcmap;
};

namespace {

struct Prof {
    cudaEvent_t a, b;
    int kind;  // 0 body, 1 compaction, 2 exchange
};

struct State {
    bool init = false;
    accmg_config cfg{};
    int P = 1, W = 1, rank = 0, V = 1;
    bool dry = false, nccl_all = false, p2p = false, use_nccl = false, chunks = false, halo_pull = false;
    std::vector<k::HaloPush> cur_push;  // per local partition: this loop's predicted-halo pushes
    accmg::Bootstrap boot;
    uint64_t* sig = nullptr;         // P2P barrier flags (W entries), mapped by every peer
    std::vector<void*> peer_sig;     // W
    std::vector<void*> sig_opened;
    uint64_t epoch = 0;
    int64_t chunk_bytes = 1 << 20;
    cudaStream_t stream = nullptr;
    accmg::NcclApi* nccl = nullptr;
    ncclComm_t comm = nullptr;
    int sticky = 0;
    std::string err = "no error";
    std::vector<accmg_region_s*> regions;
    int64_t next_id = 1;
    accmg_stats st{};
    int64_t* scratch = nullptr;     // scatter scratch
    int64_t* h_pin = nullptr;       // pinned host staging (sizes)
    int64_t* d_sizes = nullptr;     // 4*P int64 (send + all-gathered sizes)
    int* d_flag = nullptr;
    uint8_t* recv = nullptr;
    int64_t recv_cap = 0;
    // write-miss system buffers (L137): per local partition {index, value} records + counters
    // deep-halo scratch (two buffers per local partition, global-index bases)
    struct Deep {
        float* base[2] = {nullptr, nullptr};
        uint8_t* alloc[2] = {nullptr, nullptr};
        int64_t lo = 0, hi = 0;
    };
    std::vector<Deep> deep;
    std::vector<uint64_t*> miss_recs;
    int64_t miss_base = 0;
    int64_t miss_cap = 0;
    int64_t* d_miss = nullptr;       // [V] per-loop counters, [V] unused, [64] window bounds, total
    int64_t* d_miss_total = nullptr;
    // device block cache (one-process runs): blocks freed by region_destroy / hull growth are kept
    // by their allocated size and handed to the next allocation of that size (a region re-created
    // every step, as in the e2e leg, then costs no cudaMalloc / cudaFree and no device-wide sync)
    std::unordered_map<void*, size_t> blk;  // live dmalloc blocks -> allocated bytes
    std::multimap<size_t, void*> cache;     // freed blocks by size
    std::vector<Prof> prof;
    std::vector<cudaEvent_t> ev_free;
    // deferred accounting of undeclared loops whose sizes the host does not need to launch the
    // propagation (fused push): the compaction totals are copied into pinned slots on the stream
    // and booked at the next synchronising call, so the loop never waits for the device
    struct Acct {
        int64_t esize, ce;
        int slot;
        bool mc;
    };
    std::vector<Acct> pend;
    int64_t* h_acct = nullptr;  // kAcctSlots x 4 int64 (pinned)
    bool mc_ok = false;         // multicast AUTO and the node can create multicast objects
    std::string mc_why;
};
constexpr int kAcctSlots = 4096;

State S;

// pinned host staging S.h_pin (int64 slots): [0, kPinMiss) compaction sizes / all-gathered sizes
// (4 per region and partition: up to 16 regions x 64 partitions, plus the all-gather's copy), then
// 128 window bounds of the write-miss completion
constexpr int64_t kPinMiss = 4 * 16 * 64 * 2;

int fail(int code, const std::string& msg, bool sticky) {
    if (sticky && !S.sticky) S.sticky = code;
    S.err = msg;
    return code;
}

#define CUDA_TRY(x)                                                                                   \
    do {                                                                                              \
        cudaError_t e_ = (x);                                                                         \
        if (e_ != cudaSuccess) {                                                                      \
            if (e_ == cudaErrorMemoryAllocation) {                                                    \
                cudaGetLastError();                                                                   \
                return fail(ACCMG_ENOMEM, std::string(#x) + ": " + cudaGetErrorString(e_), false);  \
            }                                                                                         \
            return fail(ACCMG_ECUDA, std::string(#x) + ": " + cudaGetErrorString(e_), true);        \
        }                                                                                             \
    } while (0)

#define NCCL_TRY(x)                                                                                         \
    do {                                                                                                    \
        ncclResult_t r_ = (x);                                                                              \
        if (r_ != ncclSuccess) return fail(ACCMG_ENCCL, std::string(#x) + ": " + S.nccl->GetErrorString(r_), true); \
    } while (0)

#define TRY(x)                  \
    do {                        \
        int rc_ = (x);          \
        if (rc_ != 0) return rc_; \
    } while (0)

#define GUARD()                                                            \
    do {                                                                   \
        if (S.sticky) return S.sticky;                                     \
        if (!S.init) return fail(ACCMG_ESTATE, "accmg: not initialised", false); \
        if (!S.dry) CUDA_TRY(cudaSetDevice(S.cfg.device));                 \
    } while (0)

inline int rank_of(int g) { return g / S.V; }
inline bool local(int g) { return rank_of(g) == S.rank; }
inline int lidx(int g) { return g % S.V; }
inline int first_local() { return S.rank * S.V; }

// P2P mode: publish `mine` (this process's device allocations, one per local partition) and map
// every peer's through CUDA IPC; out[g] = pointer usable here for partition g (collective).
// Null entries publish nothing (out = nullptr).
int exchange_ptrs(const std::vector<void*>& mine, std::vector<void*>& out, std::vector<void*>& opened) {
    const int n = (int)mine.size();
    if ((size_t)n * sizeof(cudaIpcMemHandle_t) > accmg::Bootstrap::kSlotBytes)
        return fail(ACCMG_EUNSUPPORTED, "exchange_ptrs: too many handles", false);
    auto* slot = static_cast<cudaIpcMemHandle_t*>(S.boot.slot(S.rank));
    for (int i = 0; i < n; ++i) {
        if (mine[i]) CUDA_TRY(cudaIpcGetMemHandle(&slot[i], mine[i]));
        else std::memset(&slot[i], 0, sizeof(cudaIpcMemHandle_t));
    }
    std::string err;
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);
    out.assign((size_t)S.W * n, nullptr);
    for (int q = 0; q < S.W; ++q) {
        auto* qs = static_cast<cudaIpcMemHandle_t*>(S.boot.slot(q));
        for (int i = 0; i < n; ++i) {
            if (q == S.rank) {
                out[(size_t)q * n + i] = mine[i];
                continue;
            }
            cudaIpcMemHandle_t zero;
            std::memset(&zero, 0, sizeof(zero));
            if (std::memcmp(&qs[i], &zero, sizeof(zero)) == 0) continue;  // nothing allocated there
            void* p = nullptr;
            CUDA_TRY(cudaIpcOpenMemHandle(&p, qs[i], cudaIpcMemLazyEnablePeerAccess));
            out[(size_t)q * n + i] = p;
            opened.push_back(p);
        }
    }
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);  // slots may be reused after this
    return 0;
}

// P2P mode: the global barrier of L64 on the device (csrc/p2p.cu).
int dev_barrier() {
    if (!S.p2p) return 0;
    k::PtrList pl{};
    for (int q = 0; q < S.W; ++q) pl.p[pl.n++] = S.peer_sig[q];
    ++S.epoch;
    CUDA_TRY(k::device_barrier(pl, S.sig, S.rank, S.W, S.epoch, S.stream, &S.st.kernel_launches));
    return 0;
}

void chunk_of(int64_t lo, int64_t hi, int P, int g, int64_t* a, int64_t* b) {
    // L108: "the tasks in the parallel loop are equally divided among the GPUs" (reading G6)
    __int128 n = hi - lo;
    *a = lo + (int64_t)((n * g) / P);
    *b = lo + (int64_t)((n * (g + 1)) / P);
}

// Union over iterations [a, b) of the localaccess windows (L87), clipped to [0, extent).
IntervalSet window(const accmg_access& d, int64_t a, int64_t b, int64_t extent) {
    if (a >= b) return IntervalSet();
    int64_t lo = d.stride * a - d.left;
    int64_t hi = d.stride * b + d.right;  // = stride*(b-1) + stride - 1 + right + 1
    lo = std::max<int64_t>(lo, 0);
    hi = std::min<int64_t>(hi, extent);
    return IntervalSet(lo, hi);
}

// allocation granularity of the block cache: 2 MiB above 1 MiB (cudaMalloc's own page), else 512 B
size_t blk_round(size_t b) {
    return b >= ((size_t)1 << 20) ? (b + ((size_t)2 << 20) - 1) & ~(((size_t)2 << 20) - 1) : (b + 511) & ~(size_t)511;
}

void cache_release() {
    for (auto& kv : S.cache) cudaFree(kv.second);
    S.cache.clear();
}

int dmalloc(void** p, size_t bytes, bool system) {
    if (bytes == 0) bytes = 16;
    const size_t rb = blk_round(bytes);
    void* q = nullptr;
    if (S.W == 1) {
        auto it = S.cache.find(rb);
        if (it != S.cache.end()) {
            q = it->second;
            S.cache.erase(it);
        }
    }
    if (!q) {
        cudaError_t e = cudaMalloc(&q, rb);
        if (e == cudaErrorMemoryAllocation && !S.cache.empty()) {  // give the cached blocks back, retry
            cudaGetLastError();
            cache_release();
            e = cudaMalloc(&q, rb);
        }
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(ACCMG_ENOMEM, std::string("cudaMalloc(") + std::to_string(bytes) + "): " + cudaGetErrorString(e),
                        false);
        }
    }
    S.blk[q] = rb;
    *p = q;
    (system ? S.st.device_bytes_system : S.st.device_bytes_user) += (int64_t)bytes;
    return 0;
}

void dfree(void* p, size_t bytes, bool system) {
    if (!p) return;
    auto it = S.blk.find(p);
    const size_t rb = it != S.blk.end() ? it->second : 0;
    if (it != S.blk.end()) S.blk.erase(it);
    if (S.W == 1 && rb) {
        // the block's last users are on the library stream; the next owner may start with a copy on
        // another stream, so drain it (cudaFree would have synchronised the whole device)
        cudaStreamSynchronize(S.stream);
        S.cache.emplace(rb, p);
    } else {
        cudaFree(p);
    }
    (system ? S.st.device_bytes_system : S.st.device_bytes_user) -= (int64_t)bytes;
}

cudaEvent_t ev_get() {
    if (!S.ev_free.empty()) {
        cudaEvent_t e = S.ev_free.back();
        S.ev_free.pop_back();
        return e;
    }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
}

// A loop phase: an NVTX range on the host (nsys / ncu timelines) and, with profiling on, a pair of
// CUDA events on the library stream (the per-phase times of accmg_get_stats).
struct ProfScope {
    int kind;
    cudaEvent_t a = nullptr;
    explicit ProfScope(int kd) : kind(kd) {
        static const char* const kNames[3] = {"accmg body", "accmg compaction", "accmg exchange"};
        nvtxRangePushA(kNames[kd < 0 || kd > 2 ? 2 : kd]);
        if (S.cfg.profile && !S.dry) {
            a = ev_get();
            cudaEventRecord(a, S.stream);
        }
    }
    ~ProfScope() {
        if (a) {
            cudaEvent_t b = ev_get();
            cudaEventRecord(b, S.stream);
            S.prof.push_back({a, b, kind});
        }
        nvtxRangePop();
    }
};

// Host-side NVTX range for the ABI calls (loop launch, region create / destroy, sync to host).
struct NvtxScope {
    explicit NvtxScope(const char* n) { nvtxRangePushA(n); }
    ~NvtxScope() { nvtxRangePop(); }
};

// Bytes of one partition's packet of undeclared writes (runs, elements, dirty chunks), delivered to
// the P-1 other partitions (reading W8; booked by the sending process).
void book_packet(int64_t runs, int64_t elems, int64_t chunks, int64_t es, int64_t ce, bool multi, bool mc = false) {
    const int64_t hdr = 16 + 16 * runs, pay = es * elems;
    S.st.bytes_undeclared_headers += (S.P - 1) * hdr;
    S.st.bytes_undeclared_payload += (S.P - 1) * pay;
    S.st.bytes_interpartition += (S.P - 1) * (hdr + pay);
    S.st.bytes_paper_protocol += (S.P - 1) * chunks * (ce * es + ce / 8);
    if (multi) S.st.bytes_remote += (int64_t)(S.W - 1 + (S.nccl_all ? 1 : 0)) * (hdr + pay);
    if (S.p2p) S.st.bytes_remote += (int64_t)(S.P - S.V) * (hdr + pay);
    if (multi) {  // packets to the other ranks, payload stores into this rank's other replicas
        const int64_t nr = (int64_t)(S.W - 1 + (S.nccl_all ? 1 : 0)) * (hdr + pay);
        S.st.bytes_link += nr + (int64_t)(S.V - 1) * pay;
        S.st.bytes_link_remote += nr;
    } else if (mc) {  // one multimem store per dirty element; the switch replicates it
        S.st.bytes_link += pay;
        S.st.bytes_link_remote += pay;
        S.st.bytes_multicast += pay;
    } else {      // the write pass stores each dirty element into the P-1 other replicas
        S.st.bytes_link += (int64_t)(S.P - 1) * pay;
        if (S.p2p) S.st.bytes_link_remote += (int64_t)(S.P - S.V) * pay;
    }
}

// Books the deferred packets (one stream synchronisation for all loops since the last call).
int flush_acct() {
    if (S.pend.empty()) return 0;
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    for (auto& a : S.pend) {
        const int64_t* v = S.h_acct + 4 * a.slot;
        if (v[3] != v[0]) {
            S.pend.clear();
            return fail(ACCMG_ECUDA, "compaction: run starts != run ends", true);
        }
        book_packet(v[0], v[1], v[2], a.esize, a.ce, false, a.mc);
    }
    S.pend.clear();
    return 0;
}

int collect_prof() {
    TRY(flush_acct());
    if (S.prof.empty()) return 0;
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    for (auto& p : S.prof) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, p.a, p.b);
        (p.kind == 0 ? S.st.ms_body : p.kind == 1 ? S.st.ms_compact : S.st.ms_exchange) += ms;
        S.ev_free.push_back(p.a);
        S.ev_free.push_back(p.b);
    }
    S.prof.clear();
    return 0;
}

// ---- §8 row f3: VMM replicas shared through descriptors, NVLS multicast binding --------------------
// Collective (every rank takes the same decision: it depends on the config, the global validity
// tables and the init-time probe). Allocates the whole region on every rank as a driver-VMM
// allocation, maps every peer's replica here from its exported descriptor, and, with multicast
// available, binds all replicas to one multicast object (rank 0 creates it) mapped at mcmap.
int setup_vmm_region(accmg_region_s* r) {
    std::string err;
    const bool want_mc = S.cfg.multicast == ACCMG_MC_AUTO && S.mc_ok;
    const size_t bytes = accmg::vmm::round_up(S.cfg.device, (size_t)(r->extent * r->esize), want_mc);
    int fd = -1;
    if (accmg::vmm::alloc(S.cfg.device, bytes, &r->vphys, &err) != 0 || accmg::vmm::export_fd(r->vphys, &fd, &err) != 0)
        return fail(ACCMG_ECUDA, "multicast replica: " + err, true);
    std::vector<int> fds((size_t)S.W, -1);
    const bool shared = S.boot.allgather_fds(&fd, 1, fds.data(), &err);
    ::close(fd);
    if (!shared) return fail(ACCMG_ESTATE, err, true);
    r->vpeer.assign((size_t)S.W, accmg::vmm::Map{});
    for (int q = 0; q < S.W; ++q) {
        if (q == S.rank) continue;
        if (accmg::vmm::import_map(S.cfg.device, fds[q], bytes, &r->vpeer[q], &err) != 0)
            return fail(ACCMG_ECUDA, "multicast replica: " + err, true);
    }
    r->vmm = true;
    r->dev[0] = static_cast<uint8_t*>(r->vphys.ptr);
    r->abase[0] = r->dev[0];
    for (int g = 0; g < S.P; ++g) {
        r->arange[g] = Ival{0, r->extent};
        r->gdev[g] = g == S.rank ? r->dev[0] : static_cast<uint8_t*>(r->vpeer[g].ptr);
    }
    S.st.device_bytes_user += (int64_t)bytes;
    if (!want_mc) return 0;
    // the multicast object: rank 0 creates and exports it; its status travels in rank 0's slot
    int* flag = static_cast<int*>(S.boot.slot(0));
    int mfd = -1;
    if (S.rank == 0) {
        const bool ok = accmg::vmm::mc_create(S.W, bytes, &r->mc, &err) == 0 && accmg::vmm::mc_export_fd(r->mc, &mfd, &err) == 0;
        *flag = ok ? 1 : 0;
        if (!ok) S.mc_why = err;
    }
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);
    const bool created = *flag == 1;
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);  // the slot may be reused after this
    if (!created) return 0;  // unicast pushes into the shared VMM replicas
    int send = S.rank == 0 ? mfd : ::open("/dev/null", O_RDONLY | O_CLOEXEC);  // placeholder descriptor
    std::vector<int> mfds((size_t)S.W, -1);
    const bool got = S.boot.allgather_fds(&send, 1, mfds.data(), &err);
    ::close(send);
    if (!got) return fail(ACCMG_ESTATE, err, true);
    for (int q = 1; q < S.W; ++q)
        if (q != S.rank && mfds[q] >= 0) ::close(mfds[q]);
    if (S.rank != 0 && accmg::vmm::mc_import(mfds[0], &r->mc, &err) != 0)
        return fail(ACCMG_ECUDA, "multicast: " + err, true);
    if (accmg::vmm::mc_add_device(r->mc, S.cfg.device, &err) != 0) return fail(ACCMG_ECUDA, "multicast: " + err, true);
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);  // every device added before any bind
    if (accmg::vmm::mc_bind(r->mc, r->vphys, &err) != 0) return fail(ACCMG_ECUDA, "multicast: " + err, true);
    if (accmg::vmm::mc_map(S.cfg.device, r->mc, bytes, &r->mcmap, &err) != 0)
        return fail(ACCMG_ECUDA, "multicast: " + err, true);
    if (!S.boot.barrier(&err)) return fail(ACCMG_ESTATE, err, true);
    S.st.multicast_regions += 1;
    return 0;
}

void free_vmm_region(accmg_region_s* r) {
    std::string err;
    for (auto& m : r->vpeer) accmg::vmm::release(&m);
    if (r->mcmap.ptr) accmg::vmm::unmap_only(&r->mcmap);
    accmg::vmm::mc_release(r->mc, S.cfg.device, r->vphys.bytes, r->mc != 0);
    r->mc = 0;
    S.boot.barrier(&err);  // no peer still maps this replica
    S.st.device_bytes_user -= (int64_t)r->vphys.bytes;
    accmg::vmm::release(&r->vphys);
    r->abase.assign(r->abase.size(), nullptr);
    r->vmm = false;
}

// ---- window-sized replicas (§8 row f4) -------------------------------------------------------------
// Grows every partition's allocated hull to cover need[g] (the same decision on every rank: the
// tables are global). Local growth: allocate the new hull, copy what is valid, free the old one
// (after the P2P re-exchange, so no peer still maps it). P2P: re-publish the region's replicas.
// `pad`: elements added on each side of a new or grown hull (one declared stride: a write window
// that later loops read with a one-iteration halo then needs no reallocation).
int ensure_alloc(accmg_region_s* r, const std::vector<IntervalSet>& need, int64_t pad = 0) {
    if (S.dry) return 0;
    bool changed = false;
    std::vector<uint8_t*> to_free;
    std::vector<int64_t> freed_bytes;
    for (int g = 0; g < S.P; ++g) {
        if (need[g].empty()) continue;
        Ival& a = r->arange[g];
        int64_t lo = need[g].items().front().lo, hi = need[g].items().back().hi;
        if (a.hi > a.lo && lo >= a.lo && hi <= a.hi) continue;  // covered
        lo = std::max<int64_t>(lo - pad, 0);
        hi = std::min<int64_t>(hi + pad, r->extent);
        if (a.hi > a.lo) {
            lo = std::min(lo, a.lo);
            hi = std::max(hi, a.hi);
        }
        changed = true;
        const Ival old = a;
        a = {lo, hi};
        if (!local(g)) continue;
        const int li = lidx(g);
        uint8_t* nb = nullptr;
        TRY(dmalloc((void**)&nb, (size_t)((hi - lo) * r->esize), false));
        uint8_t* nbase = nb - lo * r->esize;
        if (r->abase[li]) {
            IntervalSet keep = r->valid[g].intersect(IntervalSet(old.lo, old.hi));
            for (auto& iv : keep.items())
                CUDA_TRY(cudaMemcpyAsync(nbase + iv.lo * r->esize, r->dev[li] + iv.lo * r->esize,
                                         (size_t)((iv.hi - iv.lo) * r->esize), cudaMemcpyDeviceToDevice, S.stream));
            to_free.push_back(r->abase[li]);
            freed_bytes.push_back((old.hi - old.lo) * r->esize);
        }
        r->abase[li] = nb;
        r->dev[li] = nbase;
    }
    if (changed && S.p2p) {
        // drain this process's stream first: the hull copies above must be complete before a peer
        // can reach the new replica (it may pull from or push into it right after the exchange),
        // and the previous loop's pulls and pushes through the old mappings must be finished
        // before those mappings close (every rank takes this branch: the tables are global)
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        for (auto p : r->opened) cudaIpcCloseMemHandle(p);
        r->opened.clear();
        std::vector<void*> mine(r->abase.begin(), r->abase.end()), all;
        TRY(exchange_ptrs(mine, all, r->opened));
        r->gdev.assign(S.P, nullptr);
        for (int g = 0; g < S.P; ++g)
            if (all[g]) r->gdev[g] = static_cast<uint8_t*>(all[g]) - r->arange[g].lo * r->esize;
    }
    if (!to_free.empty()) {
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        for (size_t i = 0; i < to_free.size(); ++i) dfree(to_free[i], freed_bytes[i], false);
    }
    return 0;
}

// ---- transfers between partitions (data loader pulls) -----------------------------------------
struct Xfer {
    accmg_region_s* r;
    int dst, src;  // src = -1: the host copy of rank_of(dst)
    int64_t lo, hi;
};

// Plans the pulls that make need[g] valid on every partition g; sources are chosen from the state
// before the phase: partitions of the same process first, then other processes, ascending index;
// the host copy only for what no partition holds.
void plan_pulls(accmg_region_s* r, const std::vector<IntervalSet>& need, std::vector<Xfer>& out) {
    for (int g = 0; g < S.P; ++g) {
        IntervalSet miss = need[g];
        miss.subtract(r->valid[g]);
        if (miss.empty()) continue;
        std::vector<int> order;
        for (int h = 0; h < S.P; ++h)
            if (h != g && rank_of(h) == rank_of(g)) order.push_back(h);
        for (int h = 0; h < S.P; ++h)
            if (rank_of(h) != rank_of(g)) order.push_back(h);
        for (int h : order) {
            if (miss.empty()) break;
            IntervalSet piece = miss.intersect(r->valid[h]);
            for (auto& iv : piece.items()) out.push_back({r, g, h, iv.lo, iv.hi});
            miss.subtract(piece);
        }
        for (auto& iv : miss.items()) out.push_back({r, g, -1, iv.lo, iv.hi});
    }
}

int run_xfers(const std::vector<Xfer>& xs) {
    // accounting (partition-to-partition bytes are whole-job totals, identical on every rank)
    for (auto& x : xs) {
        int64_t nb = (x.hi - x.lo) * x.r->esize;
        if (!local(x.dst)) continue;  // bytes are counted by the receiving process
        if (x.src >= 0) {
            S.st.bytes_interpartition += nb;
            S.st.bytes_declared += nb;
            S.st.bytes_link += nb;
            if (rank_of(x.src) != rank_of(x.dst)) {
                S.st.bytes_remote += nb;
                S.st.bytes_link_remote += nb;
            }
        } else {
            S.st.bytes_h2d += nb;
            if (!x.r->host_valid.contains(IntervalSet(x.lo, x.hi)))
                return fail(ACCMG_ESTATE, "data loader: range valid on no partition and not on the host copy", false);
        }
    }
    if (S.dry || xs.empty()) return 0;
    ProfScope ps(2);
    bool any_nccl = false;
    // device-to-device pulls of this phase (same-GPU replicas, or peers' replicas mapped through IPC
    // and read over NVLink): small phases (halos) go as ONE batched copy kernel, large ones through
    // the copy engines
    k::CopyList batch{};
    int64_t batch_bytes = 0;
    std::vector<std::pair<const Xfer*, const uint8_t*>> d2d;
    for (auto& x : xs) {
        const size_t nb = (size_t)((x.hi - x.lo) * x.r->esize);
        const int64_t off = x.lo * x.r->esize;
        if (x.src < 0) {
            if (local(x.dst))
                CUDA_TRY(cudaMemcpyAsync(x.r->dev[lidx(x.dst)] + off, x.r->host + off, nb, cudaMemcpyHostToDevice,
                                         S.stream));
        } else if (local(x.src) && local(x.dst) && !S.nccl_all) {
            d2d.push_back({&x, x.r->dev[lidx(x.src)] + off});
        } else if (S.p2p) {
            if (local(x.dst)) d2d.push_back({&x, x.r->gdev[x.src] + off});
        } else if (local(x.src) || local(x.dst)) {
            any_nccl = true;
        }
    }
    for (auto& [x, src] : d2d) batch_bytes += (x->hi - x->lo) * x->r->esize;
    const bool batched = !d2d.empty() && (int)d2d.size() <= k::kMaxCopies && batch_bytes <= (64ll << 20);
    for (auto& [x, src] : d2d) {
        const size_t nb = (size_t)((x->hi - x->lo) * x->r->esize);
        uint8_t* dst = x->r->dev[lidx(x->dst)] + x->lo * x->r->esize;
        if (batched) {
            batch.dst[batch.n] = dst;
            batch.src[batch.n] = src;
            batch.bytes[batch.n] = (int64_t)nb;
            ++batch.n;
        } else {
            CUDA_TRY(cudaMemcpyAsync(dst, src, nb, cudaMemcpyDefault, S.stream));
        }
    }
    if (batched) CUDA_TRY(k::copy_batch(batch, S.stream, &S.st.kernel_launches));
    if (any_nccl) {
        NCCL_TRY(S.nccl->GroupStart());
        for (auto& x : xs) {
            if (x.src < 0) continue;
            const bool viaN = rank_of(x.src) != rank_of(x.dst) || S.nccl_all;
            if (!viaN) continue;
            const size_t nb = (size_t)((x.hi - x.lo) * x.r->esize);
            const int64_t off = x.lo * x.r->esize;
            if (local(x.src))
                NCCL_TRY(S.nccl->Send(x.r->dev[lidx(x.src)] + off, nb, ncclUint8, rank_of(x.dst), S.comm, S.stream));
            if (local(x.dst))
                NCCL_TRY(S.nccl->Recv(x.r->dev[lidx(x.dst)] + off, nb, ncclUint8, rank_of(x.src), S.comm, S.stream));
        }
        NCCL_TRY(S.nccl->GroupEnd());
    }
    return 0;
}

// ---- tracking buffers ---------------------------------------------------------------------------
int chunk_elems(const accmg_region_s* r) { return (int)std::max<int64_t>(S.chunk_bytes / r->esize, 32); }

int ensure_trk(accmg_region_s* r, int li) {
    Trk& t = r->trk[li];
    if (t.l1) return 0;
    const int64_t ce = chunk_elems(r);
    t.nwords = (r->extent + 31) / 32;
    const int64_t nchunks = (r->extent + ce - 1) / ce;
    t.nl2 = (nchunks + 31) / 32;
    t.ntiles = (t.nwords + k::kTileWords - 1) / k::kTileWords;
    TRY(dmalloc((void**)&t.l1, t.nwords * 4, true));
    TRY(dmalloc((void**)&t.l2, t.nl2 * 4, true));
    TRY(dmalloc((void**)&t.tile_counts, t.ntiles * 24, true));
    TRY(dmalloc((void**)&t.tile_offs, t.ntiles * 24, true));
    TRY(dmalloc((void**)&t.tile_edges, t.ntiles * 8, true));
    TRY(dmalloc((void**)&t.totals, 64, true));
    CUDA_TRY(cudaMemsetAsync(t.l1, 0, t.nwords * 4, S.stream));
    CUDA_TRY(cudaMemsetAsync(t.l2, 0, t.nl2 * 4, S.stream));
    if (S.cfg.debug_checks) {
        TRY(dmalloc((void**)&t.snap_l1, t.nwords * 4, true));
        TRY(dmalloc((void**)&t.snap_l2, t.nl2 * 4, true));
    }
    return 0;
}

int ensure_packed(Trk& t, int64_t bytes) {
    if (t.packed_cap >= bytes) return 0;
    int64_t cap = std::max<int64_t>(bytes, t.packed_cap + t.packed_cap / 2);
    if (t.packed) {
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        dfree(t.packed, t.packed_cap, true);
        t.packed = nullptr;
    }
    TRY(dmalloc((void**)&t.packed, cap, true));
    t.packed_cap = cap;
    return 0;
}

int ensure_recv(int64_t bytes) {
    if (S.recv_cap >= bytes) return 0;
    if (S.recv) {
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        dfree(S.recv, S.recv_cap, true);
        S.recv = nullptr;
    }
    TRY(dmalloc((void**)&S.recv, bytes, true));
    S.recv_cap = bytes;
    return 0;
}

// Scratch for the deep-halo body: element range [lo, hi) in two buffers (grow-only, system memory).
int ensure_deep(int li, int64_t lo, int64_t hi) {
    if ((int)S.deep.size() < S.V) S.deep.resize(S.V);
    auto& D = S.deep[li];
    if (D.alloc[0] && lo >= D.lo && hi <= D.hi) return 0;
    if (D.alloc[0]) {
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        lo = std::min(lo, D.lo);
        hi = std::max(hi, D.hi);
        for (int q = 0; q < 2; ++q) dfree(D.alloc[q], (D.hi - D.lo) * 4, true);
    }
    for (int q = 0; q < 2; ++q) {
        TRY(dmalloc((void**)&D.alloc[q], (size_t)(hi - lo) * 4, true));
        D.base[q] = reinterpret_cast<float*>(D.alloc[q]) - lo;
    }
    D.lo = lo;
    D.hi = hi;
    return 0;
}

k::Track track_of(accmg_region_s* r, int li, bool on) {
    k::Track t{nullptr, nullptr, 0};
    if (!on) return t;
    t.l1 = r->trk[li].l1;
    t.l2 = r->trk[li].l2;
    int sh = 0;
    while ((1ll << sh) < chunk_elems(r)) ++sh;
    t.l2_shift = sh;
    return t;
}

// ---- bodies ---------------------------------------------------------------------------------------
struct BodySpec {
    int n;
    int mode[5];
    int esize[5];
    int ndim;
    size_t args;
};

bool body_spec(int id, BodySpec* b) {
    switch (id) {
        case ACCMG_BODY_JACOBI2D_5PT: *b = {2, {ACCMG_R, ACCMG_W}, {4, 4}, 2, sizeof(accmg_args_jacobi2d)}; return true;
        case ACCMG_BODY_GEMM_BF16_F32: *b = {3, {ACCMG_R, ACCMG_R, ACCMG_W}, {2, 2, 4}, 2, sizeof(accmg_args_gemm)}; return true;
        case ACCMG_BODY_KMEANS_ASSIGN:
            *b = {5, {ACCMG_R, ACCMG_R, ACCMG_W, ACCMG_REDUCE_SUM, ACCMG_REDUCE_SUM}, {4, 4, 4, 8, 8}, 1,
                  sizeof(accmg_args_kmeans)};
            return true;
        case ACCMG_BODY_KMEANS_UPDATE:
            *b = {3, {ACCMG_RW, ACCMG_RW, ACCMG_W}, {8, 8, 4}, 1, sizeof(accmg_args_kmeans)};
            return true;
        case ACCMG_BODY_TEST_SPARSE_WRITE: *b = {2, {ACCMG_R, ACCMG_W}, {4, 4}, 1, sizeof(accmg_args_sparse)}; return true;
        case ACCMG_BODY_TEST_MASKED_WRITE:
            *b = {3, {ACCMG_R, ACCMG_R, ACCMG_W}, {4, 1, 4}, 1, sizeof(accmg_args_masked)};
            return true;
        case ACCMG_BODY_SCATTER: *b = {3, {ACCMG_R, ACCMG_R, ACCMG_W}, {4, 4, 4}, 1, sizeof(accmg_args_scatter)}; return true;
        case ACCMG_BODY_JACOBI3D_7PT: *b = {2, {ACCMG_R, ACCMG_W}, {4, 4}, 3, sizeof(accmg_args_jacobi3d)}; return true;
        case ACCMG_BODY_JACOBI2D_DEEP: *b = {2, {ACCMG_R, ACCMG_W}, {4, 4}, 2, sizeof(accmg_args_jacobi2d_deep)}; return true;
        default: return false;
    }
}

int validate_body(const accmg_bounds* bd, int body, const accmg_access* d, const void* args) {
    auto bad = [](const std::string& m) { return fail(ACCMG_EINVAL, "loop_launch: " + m, false); };
    auto ext = [&](int i) { return d[i].region->extent; };
    switch (body) {
        case ACCMG_BODY_JACOBI2D_5PT: {
            auto a = static_cast<const accmg_args_jacobi2d*>(args);
            if (a->rows < 3 || a->cols < 3) return bad("jacobi: rows, cols >= 3");
            if (ext(0) != a->rows * a->cols || ext(1) != a->rows * a->cols) return bad("jacobi: region extent != rows*cols");
            if (bd->lo[0] < 1 || bd->hi[0] > a->rows - 1 || bd->lo[1] < 1 || bd->hi[1] > a->cols - 1)
                return bad("jacobi: bounds must lie in [1,rows-1) x [1,cols-1)");
            if (d[0].region == d[1].region) return bad("jacobi: src and dst must differ");
            return 0;
        }
        case ACCMG_BODY_JACOBI2D_DEEP: {
            auto a = static_cast<const accmg_args_jacobi2d_deep*>(args);
            if (a->rows < 3 || a->cols < 3 || a->h < 1 || a->h > 64) return bad("jacobi_deep: rows, cols >= 3, 1 <= h <= 64");
            if (ext(0) != a->rows * a->cols || ext(1) != a->rows * a->cols) return bad("jacobi_deep: region extent != rows*cols");
            if (bd->lo[0] < 1 || bd->hi[0] > a->rows - 1 || bd->lo[1] < 1 || bd->hi[1] > a->cols - 1)
                return bad("jacobi_deep: bounds must lie in [1,rows-1) x [1,cols-1)");
            if (d[0].region == d[1].region) return bad("jacobi_deep: src and dst must differ");
            return 0;
        }
        case ACCMG_BODY_TEST_SPARSE_WRITE: {
            auto a = static_cast<const accmg_args_sparse*>(args);
            if (a->rows < 1 || a->cols < 1 || a->period < 1) return bad("sparse: rows, cols, period >= 1");
            if (ext(0) != a->rows * a->cols || ext(1) != a->rows * a->cols) return bad("sparse: extent != rows*cols");
            if (bd->lo[0] < 0 || bd->hi[0] > a->rows) return bad("sparse: bounds outside [0,rows)");
            if (d[0].region == d[1].region) return bad("sparse: in and out must differ");
            return 0;
        }
        case ACCMG_BODY_TEST_MASKED_WRITE: {
            auto a = static_cast<const accmg_args_masked*>(args);
            if (a->n < 1) return bad("masked: n >= 1");
            if (ext(0) != a->n || ext(1) != a->n || ext(2) != a->n) return bad("masked: extents != n");
            if (bd->lo[0] < 0 || bd->hi[0] > a->n) return bad("masked: bounds outside [0,n)");
            if (d[0].region == d[2].region) return bad("masked: in and out must differ");
            return 0;
        }
        case ACCMG_BODY_JACOBI3D_7PT: {
            auto a = static_cast<const accmg_args_jacobi3d*>(args);
            if (a->n0 < 3 || a->n1 < 3 || a->n2 < 3) return bad("jacobi3d: n0, n1, n2 >= 3");
            const int64_t E = a->n0 * a->n1 * a->n2;
            if (ext(0) != E || ext(1) != E) return bad("jacobi3d: region extent != n0*n1*n2");
            if (bd->lo[0] < 1 || bd->hi[0] > a->n0 - 1 || bd->lo[1] < 1 || bd->hi[1] > a->n1 - 1 || bd->lo[2] < 1 ||
                bd->hi[2] > a->n2 - 1)
                return bad("jacobi3d: bounds must lie in the interior");
            if (d[0].region == d[1].region) return bad("jacobi3d: src and dst must differ");
            if (a->n2 % 4 != 0) return fail(ACCMG_EUNSUPPORTED, "jacobi3d: needs n2 % 4 == 0", false);
            return 0;
        }
        case ACCMG_BODY_SCATTER: {
            auto a = static_cast<const accmg_args_scatter*>(args);
            if (a->n < 1 || a->m < 1) return bad("scatter: n, m >= 1");
            if (ext(0) != a->n || ext(1) != a->n || ext(2) != a->m) return bad("scatter: extents");
            if (bd->lo[0] < 0 || bd->hi[0] > a->n) return bad("scatter: bounds outside [0,n)");
            if (!d[2].declared)
                return fail(ACCMG_EUNSUPPORTED, "scatter: dst must be a distributed (declared) array", false);
            if (S.use_nccl && S.W > 1)
                return fail(ACCMG_EUNSUPPORTED, "scatter: write misses need the P2P transport", false);
            return 0;
        }
        case ACCMG_BODY_GEMM_BF16_F32: {
            auto a = static_cast<const accmg_args_gemm*>(args);
            if (a->M < 1 || a->N < 1 || a->K < 1) return bad("gemm: M, N, K >= 1");
            if (ext(0) != a->M * a->K || ext(1) != a->K * a->N || ext(2) != a->M * a->N) return bad("gemm: extents");
            if (bd->lo[0] < 0 || bd->hi[0] > a->M || bd->lo[1] != 0 || bd->hi[1] != a->N)
                return bad("gemm: bounds must be rows within [0,M) x all of [0,N)");
            if (a->N % 8 != 0 || a->K % 64 != 0) return fail(ACCMG_EUNSUPPORTED, "gemm: needs N % 8 == 0, K % 64 == 0", false);
            return 0;
        }
        case ACCMG_BODY_KMEANS_ASSIGN:
        case ACCMG_BODY_KMEANS_UPDATE: {
            auto a = static_cast<const accmg_args_kmeans*>(args);
            if (a->n < 1 || a->d < 1 || a->k < 1 || a->shift < ACCMG_KMEANS_EXACT || a->shift > 30)
                return bad("kmeans: n, d, k >= 1, shift in [0,30] or ACCMG_KMEANS_EXACT");
            const bool exact = a->shift == ACCMG_KMEANS_EXACT;
            if (exact ? (a->d > 64 || a->k > 1024 || (int64_t)a->k * a->d > 16384) : (a->d > 32 || a->k > 1024))
                return fail(ACCMG_EUNSUPPORTED, "kmeans: d <= 32, k <= 1024 (exact mode: d <= 64, k*d <= 16384)", false);
            // exact mode: the sums region holds ACCMG_KMEANS_WINDOWS int64 windows per (cluster, dim)
            const int64_t sum_ext = (int64_t)a->k * a->d * (exact ? ACCMG_KMEANS_WINDOWS : 1);
            if (body == ACCMG_BODY_KMEANS_ASSIGN) {
                if (ext(0) != a->n * a->d || ext(1) != (int64_t)a->k * a->d || ext(2) != a->n ||
                    ext(3) != sum_ext || ext(4) != a->k)
                    return bad("kmeans_assign: extents");
                if (bd->lo[0] < 0 || bd->hi[0] > a->n) return bad("kmeans_assign: bounds outside [0,n)");
            } else {
                if (ext(0) != sum_ext || ext(1) != a->k || ext(2) != (int64_t)a->k * a->d)
                    return bad("kmeans_update: extents");
                if (bd->lo[0] < 0 || bd->hi[0] > a->k) return bad("kmeans_update: bounds outside [0,k)");
            }
            return 0;
        }
    }
    return bad("unknown body");
}

int launch_body(int body, const accmg_bounds* bd, const accmg_access* d, const void* args, int g, int64_t a,
                int64_t b, const std::vector<bool>& tracked) {
    const int li = lidx(g);
    auto P = [&](int i) { return d[i].region->dev[li]; };
    auto T = [&](int i) { return track_of(d[i].region, li, tracked[i]); };
    cudaError_t e = cudaSuccess;
    int64_t* L = &S.st.kernel_launches;
    switch (body) {
        case ACCMG_BODY_JACOBI2D_5PT: {
            auto x = static_cast<const accmg_args_jacobi2d*>(args);
            const Ival al = d[0].region->arange[g];
            e = k::jacobi2d((const float*)P(0), (float*)P(1), x->rows, x->cols, a, b, bd->lo[1], bd->hi[1], al.lo, al.hi,
                            T(1), 0, S.stream, L, S.cur_push[li]);
            break;
        }
        case ACCMG_BODY_JACOBI2D_DEEP: {
            // h sweeps: src -> tmp -> tmp' -> ... -> dst over shrinking row ranges; the scratch
            // buffers hold rows [a-h, b+h) (global-index bases) with src's fixed frame
            auto x = static_cast<const accmg_args_jacobi2d_deep*>(args);
            const int64_t C = x->cols, h = x->h, rlo = bd->lo[0], rhi = bd->hi[0];
            const int64_t lo = std::max<int64_t>(a - h, 0), hi = std::min<int64_t>(b + h, x->rows);
            const Ival al = d[0].region->arange[g];
            if (h > 1) {  // fused: h sweeps per launch without scratch (register-streamed levels)
                e = k::jacobi2d_deep_stream((const float*)P(0), (float*)P(1), x->rows, C, a, b, rlo, rhi, bd->lo[1], bd->hi[1], (int)h,
                          al.lo, al.hi, T(1), S.stream, L);
                if (e != cudaErrorNotSupported) break;
                e = cudaSuccess;
            }
            TRY(ensure_deep(li, lo * C, hi * C));
            float* tmp[2] = {S.deep[li].base[0], S.deep[li].base[1]};
            if (h > 1) {
                for (int q = 0; q < 2; ++q)
                    CUDA_TRY(k::frame_copy((const float*)P(0), tmp[q], C, lo, hi, rlo, rhi, bd->lo[1], bd->hi[1], S.stream, L));
            }
            const float* in = (const float*)P(0);
            int64_t in_lo = al.lo, in_hi = al.hi;
            for (int64_t kk = 1; kk <= h && e == cudaSuccess; ++kk) {
                const bool last = kk == h;
                float* out = last ? (float*)P(1) : tmp[kk % 2];
                const int64_t r0 = std::max<int64_t>(a - (h - kk), rlo), r1 = std::min<int64_t>(b + (h - kk), rhi);
                e = k::jacobi2d(in, out, x->rows, C, r0, r1, bd->lo[1], bd->hi[1], in_lo, in_hi, last ? T(1) : k::Track{},
                                0, S.stream, L);
                in = out;
                in_lo = lo * C;
                in_hi = hi * C;
            }
            break;
        }
        case ACCMG_BODY_TEST_SPARSE_WRITE: {
            auto x = static_cast<const accmg_args_sparse*>(args);
            e = k::sparse_rows((const float*)P(0), (float*)P(1), x->rows, x->cols, a, b, x->period, T(1), S.stream, L);
            break;
        }
        case ACCMG_BODY_TEST_MASKED_WRITE:
            e = k::masked_write((const float*)P(0), (const uint8_t*)P(1), (float*)P(2), a, b, T(2), S.stream, L);
            break;
        case ACCMG_BODY_JACOBI3D_7PT: {
            auto x = static_cast<const accmg_args_jacobi3d*>(args);
            const Ival al = d[0].region->arange[g];
            e = k::jacobi3d((const float*)P(0), (float*)P(1), x->n0, x->n1, x->n2, a, b, bd->lo[1], bd->hi[1],
                            bd->lo[2], bd->hi[2], al.lo, al.hi, T(1), S.stream, L);
            break;
        }
        case ACCMG_BODY_SCATTER: {
            IntervalSet w = window(d[2], a, b, d[2].region->extent);
            const int64_t wlo = w.empty() ? 0 : w.items()[0].lo, whi = w.empty() ? 0 : w.items()[0].hi;
            e = k::scatter_body((const float*)P(0), (const int32_t*)P(1), (float*)P(2), a, b, wlo, whi,
                                S.miss_recs[li], S.d_miss + li, S.stream, L);
            break;
        }
        case ACCMG_BODY_GEMM_BF16_F32: {
            auto x = static_cast<const accmg_args_gemm*>(args);
            e = k::gemm_bf16((const uint16_t*)P(0), (const uint16_t*)P(1), (float*)P(2), x->M, x->N, x->K, a, b,
                             d[0].region->arange[g].lo, S.stream, L);
            break;
        }
        case ACCMG_BODY_KMEANS_ASSIGN: {
            auto x = static_cast<const accmg_args_kmeans*>(args);
            e = k::kmeans_assign((const float*)P(0), (const float*)P(1), (int32_t*)P(2), d[3].region->partial[li],
                                 d[4].region->partial[li], a, b, x->d, x->k, x->shift, S.d_flag + 1, S.stream, L);
            break;
        }
        case ACCMG_BODY_KMEANS_UPDATE: {
            auto x = static_cast<const accmg_args_kmeans*>(args);
            e = k::kmeans_update((int64_t*)P(0), (int64_t*)P(1), (float*)P(2), a, b, x->d, x->shift, T(0), T(1), T(2),
                                 S.stream, L);
            break;
        }
    }
    if (e == cudaErrorNotSupported) return fail(ACCMG_EUNSUPPORTED, "body not supported on this build/shape", false);
    CUDA_TRY(e);
    S.st.body_launches += 1;
    return 0;
}

// ---- coherence of undeclared writes (L129-135) -----------------------------------------------------
// Every replica of r other than local partition li's: the local ones and (P2P mode) the peers'
// replicas through their IPC mappings over NVLink.
k::PtrList push_list(accmg_region_s* r, int li) {
    const int g = first_local() + li;
    k::PtrList dl{};
    if (r->mcmap.ptr) {  // NVLS: one multicast address for all replicas (global-index base)
        dl.p[0] = r->mcmap.ptr;
        dl.n = 1;
        dl.mc = 1;
        return dl;
    }
    if (S.p2p) {
        for (int h = 0; h < S.P; ++h)
            if (h != g) dl.p[dl.n++] = r->gdev[h];
    } else {
        for (int h = 0; h < S.V; ++h)
            if (h != li) dl.p[dl.n++] = r->dev[h];
    }
    return dl;
}

int propagate_dirty(const std::vector<accmg_region_s*>& regs) {
    // with the fused push nothing on the host needs the packet sizes before the write pass (the
    // packed buffer is not materialised): the loop does not synchronise, the sizes are booked later
    const bool fused = !S.use_nccl;
    const bool deferred = fused && !S.cfg.debug_checks && !S.chunks;
    if (deferred && S.pend.size() + regs.size() * S.V > (size_t)kAcctSlots) TRY(flush_acct());
    // 1. per local replica: (debug snapshot), count, scan
    {
        ProfScope ps(1);
        for (auto* r : regs)
            for (int li = 0; li < S.V; ++li) {
                Trk& t = r->trk[li];
                if (S.cfg.debug_checks) {
                    CUDA_TRY(cudaMemcpyAsync(t.snap_l1, t.l1, t.nwords * 4, cudaMemcpyDeviceToDevice, S.stream));
                    CUDA_TRY(cudaMemcpyAsync(t.snap_l2, t.l2, t.nl2 * 4, cudaMemcpyDeviceToDevice, S.stream));
                    t.has_snap = true;
                }
                int cw = 0;
                while ((1ll << cw) < chunk_elems(r) / 32) ++cw;
                CUDA_TRY(k::compact_count(t.l1, t.l2, t.nwords, cw, t.ntiles, t.tile_counts, t.tile_edges, S.stream,
                                          &S.st.kernel_launches));
                if (S.chunks) {
                    // the paper's protocol: dirty chunks merged into every peer by their L1 bits
                    ProfScope px(2);
                    const int g = first_local() + li;
                    k::PtrList dl{};
                    for (int h = 0; h < S.P; ++h)
                        if (h != g) dl.p[dl.n++] = S.p2p ? (void*)r->gdev[h] : (void*)r->dev[lidx(h)];
                    CUDA_TRY(k::chunk_merge(t.l1, t.l2, t.nwords, cw, r->dev[li], (int)r->esize, dl, S.stream,
                                            &S.st.kernel_launches));
                }
                CUDA_TRY(k::compact_scan(t.tile_counts, t.ntiles, t.tile_offs, t.totals, t.l2, t.nl2, S.stream,
                                         &S.st.kernel_launches));
            }
        if (S.cfg.debug_checks) {
            CUDA_TRY(cudaMemsetAsync(S.d_flag, 0, sizeof(int), S.stream));
            for (auto* r : regs)
                for (int a = 0; a < S.V; ++a)
                    for (int b = a + 1; b < S.V; ++b)
                        CUDA_TRY(k::bitmap_overlap(r->trk[a].snap_l1, r->trk[b].snap_l1, r->trk[a].nwords, S.d_flag,
                                                   S.stream, &S.st.kernel_launches));
        }
    }
    if (deferred) {
        ProfScope ps(1);
        for (auto* r : regs)
            for (int li = 0; li < S.V; ++li) {
                Trk& t = r->trk[li];
                const int slot = (int)S.pend.size();
                CUDA_TRY(cudaMemcpyAsync(S.h_acct + 4 * slot, t.totals, 32, cudaMemcpyDeviceToHost, S.stream));
                S.pend.push_back({r->esize, chunk_elems(r), slot, r->mcmap.ptr != nullptr});
                CUDA_TRY(k::compact_write(t.l1, t.nwords, r->extent, t.ntiles, t.tile_counts, t.tile_offs, t.tile_edges,
                                          r->dev[li], (int)r->esize, nullptr, 0, push_list(r, li), S.stream,
                                          &S.st.kernel_launches, 0));
                t.has_packed = false;
            }
        return 0;
    }
    // 2. sizes to the host (one synchronisation for all regions); with the P2P transport (or one
    // process) the write pass also pushes every dirty element into the other replicas, so the
    // packed buffer is not re-read by a separate scatter pass
    int slot = 0;
    for (auto* r : regs)
        for (int li = 0; li < S.V; ++li, ++slot)
            CUDA_TRY(cudaMemcpyAsync(S.h_pin + 4 * slot, r->trk[li].totals, 32, cudaMemcpyDeviceToHost, S.stream));
    if (S.cfg.debug_checks)
        CUDA_TRY(cudaMemcpyAsync((int*)(S.h_pin + 4 * slot), S.d_flag, sizeof(int), cudaMemcpyDeviceToHost, S.stream));
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    if (S.cfg.debug_checks && *(int*)(S.h_pin + 4 * slot))
        return fail(ACCMG_ECONFLICT, "two partitions wrote the same replicated element (L62: no dependences)", false);
    slot = 0;
    for (auto* r : regs)
        for (int li = 0; li < S.V; ++li, ++slot) {
            Trk& t = r->trk[li];
            t.n_runs = S.h_pin[4 * slot];
            t.n_elems = S.h_pin[4 * slot + 1];
            t.dirty_chunks = S.h_pin[4 * slot + 2];
            if (S.h_pin[4 * slot + 3] != t.n_runs) return fail(ACCMG_ECUDA, "compaction: run starts != run ends", true);
            t.packed_bytes = 16 + 16 * t.n_runs + r->esize * t.n_elems;
            if (S.chunks) continue;  // merged already; nothing to pack
            // the canonical packed buffer is materialised only when something reads it: the
            // message-passing transport, the separate scatter pass, or debug inspection; with the
            // fused push the write pass stores each dirty element into the other replicas only
            const bool keep = !fused || S.cfg.debug_checks;
            if (keep) {
                TRY(ensure_packed(t, t.packed_bytes));
                CUDA_TRY(cudaMemcpyAsync(t.packed, t.totals, 16, cudaMemcpyDeviceToDevice, S.stream));
            }
            ProfScope ps(1);
            k::PtrList push{};
            if (fused) push = push_list(r, li);
            CUDA_TRY(k::compact_write(t.l1, t.nwords, r->extent, t.ntiles, t.tile_counts, t.tile_offs, t.tile_edges, r->dev[li],
                                      (int)r->esize, keep ? t.packed : nullptr, t.n_runs, push, S.stream,
                                      &S.st.kernel_launches, keep ? 1 : 0));
            t.has_packed = keep;
        }
    // 3. sizes of every partition's packet (all-gather across processes when needed)
    std::vector<int64_t> runs(S.P * regs.size()), elems(S.P * regs.size()), chunks(S.P * regs.size());
    const bool multi = S.use_nccl;  // packets travel through NCCL (sizes must be all-gathered)
    if (multi) {
        // layout per rank: [region][local] x {runs, elems, chunks, pad}
        const int64_t per = (int64_t)regs.size() * S.V * 4;
        slot = 0;
        for (auto* r : regs)
            for (int li = 0; li < S.V; ++li, ++slot) {
                S.h_pin[4 * slot] = r->trk[li].n_runs;
                S.h_pin[4 * slot + 1] = r->trk[li].n_elems;
                S.h_pin[4 * slot + 2] = r->trk[li].dirty_chunks;
                S.h_pin[4 * slot + 3] = 0;
            }
        CUDA_TRY(cudaMemcpyAsync(S.d_sizes, S.h_pin, per * 8, cudaMemcpyHostToDevice, S.stream));
        NCCL_TRY(S.nccl->AllGather(S.d_sizes, S.d_sizes + per, per, ncclInt64, S.comm, S.stream));
        CUDA_TRY(cudaMemcpyAsync(S.h_pin, S.d_sizes + per, per * S.W * 8, cudaMemcpyDeviceToHost, S.stream));
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        for (int q = 0; q < S.W; ++q)
            for (size_t ri = 0; ri < regs.size(); ++ri)
                for (int li = 0; li < S.V; ++li) {
                    const int64_t* v = S.h_pin + q * per + 4 * (ri * S.V + li);
                    const int g = q * S.V + li;
                    runs[ri * S.P + g] = v[0];
                    elems[ri * S.P + g] = v[1];
                    chunks[ri * S.P + g] = v[2];
                }
    } else {
        for (size_t ri = 0; ri < regs.size(); ++ri)
            for (int li = 0; li < S.V; ++li) {
                const int g = first_local() + li;
                runs[ri * S.P + g] = regs[ri]->trk[li].n_runs;
                elems[ri * S.P + g] = regs[ri]->trk[li].n_elems;
                chunks[ri * S.P + g] = regs[ri]->trk[li].dirty_chunks;
            }
    }
    if (S.chunks) {
        // accounting of the paper's protocol: every dirty chunk (data + its L1 bits) to P-1 peers
        for (size_t ri = 0; ri < regs.size(); ++ri) {
            const int64_t es = regs[ri]->esize, ce = chunk_elems(regs[ri]);
            for (int li = 0; li < S.V; ++li) {
                const int64_t nb = (S.P - 1) * regs[ri]->trk[li].dirty_chunks * (ce * es + ce / 8);
                S.st.bytes_interpartition += nb;
                S.st.bytes_paper_protocol += nb;
                S.st.bytes_undeclared_payload += (S.P - 1) * regs[ri]->trk[li].dirty_chunks * ce * es;
                S.st.bytes_undeclared_headers += (S.P - 1) * regs[ri]->trk[li].dirty_chunks * (ce / 8);
                if (S.p2p) S.st.bytes_remote += (int64_t)(S.P - S.V) * regs[ri]->trk[li].dirty_chunks * (ce * es + ce / 8);
                // the merge kernel reads the chunk bits locally and stores only the dirty elements
                S.st.bytes_link += (int64_t)(S.P - 1) * regs[ri]->trk[li].n_elems * es;
                if (S.p2p) S.st.bytes_link_remote += (int64_t)(S.P - S.V) * regs[ri]->trk[li].n_elems * es;
            }
        }
        return 0;
    }
    // accounting (by the sending process): every packet is delivered to the P-1 other partitions
    // (reading W8)
    for (size_t ri = 0; ri < regs.size(); ++ri)
        for (int g = 0; g < S.P; ++g)
            if (local(g))
                book_packet(runs[ri * S.P + g], elems[ri * S.P + g], chunks[ri * S.P + g], regs[ri]->esize,
                            chunk_elems(regs[ri]), multi, regs[ri]->mcmap.ptr != nullptr);
    // 4. exchange + scatter
    ProfScope ps(2);
    if (!multi) return 0;  // pushed into every other replica by the write pass
    // receive every packet that comes from another process (or, in NCCL_ALL mode, from anyone) once
    int64_t need = 0;
    std::vector<int64_t> roff(S.P * regs.size(), -1);
    for (size_t ri = 0; ri < regs.size(); ++ri)
        for (int g = 0; g < S.P; ++g) {
            if (local(g) && !S.nccl_all) continue;
            roff[ri * S.P + g] = need;
            need += (16 + 16 * runs[ri * S.P + g] + regs[ri]->esize * elems[ri * S.P + g] + 255) / 256 * 256;
        }
    TRY(ensure_recv(need));
    NCCL_TRY(S.nccl->GroupStart());
    for (size_t ri = 0; ri < regs.size(); ++ri)
        for (int g = 0; g < S.P; ++g) {
            const size_t nb = (size_t)(16 + 16 * runs[ri * S.P + g] + regs[ri]->esize * elems[ri * S.P + g]);
            if (local(g))
                for (int q = 0; q < S.W; ++q)
                    if (q != S.rank || S.nccl_all)
                        NCCL_TRY(S.nccl->Send(regs[ri]->trk[lidx(g)].packed, nb, ncclUint8, q, S.comm, S.stream));
            if (roff[ri * S.P + g] >= 0)
                NCCL_TRY(S.nccl->Recv(S.recv + roff[ri * S.P + g], nb, ncclUint8, rank_of(g), S.comm, S.stream));
        }
    NCCL_TRY(S.nccl->GroupEnd());
    for (size_t ri = 0; ri < regs.size(); ++ri) {
        accmg_region_s* r = regs[ri];
        for (int g = 0; g < S.P; ++g) {
            k::PtrList dl{};
            for (int h = 0; h < S.V; ++h)
                if (first_local() + h != g) dl.p[dl.n++] = r->dev[h];
            const uint8_t* src = roff[ri * S.P + g] >= 0 ? S.recv + roff[ri * S.P + g] : r->trk[lidx(g)].packed;
            if (roff[ri * S.P + g] < 0 && !local(g)) continue;
            CUDA_TRY(k::scatter_packed(src, runs[ri * S.P + g], dl, (int)r->esize, S.scratch, S.stream,
                                       &S.st.kernel_launches));
        }
    }
    return 0;
}

// ---- reductiontoarray merge (L112: block -> GPU -> across GPUs) ------------------------------------
int merge_reduce(accmg_region_s* r) {
    ProfScope ps(2);
    if (S.p2p) {
        // every rank sums all P partials (its own and its peers', read over NVLink) after a
        // barrier, applies the total to its replicas, and a second barrier keeps the partials
        // alive until every rank has read them
        TRY(dev_barrier());
        CUDA_TRY(cudaMemsetAsync(r->acc, 0, r->extent * 8, S.stream));
        k::PtrList src{};
        for (int g = 0; g < S.P; ++g) src.p[src.n++] = r->gpartial[g];
        CUDA_TRY(k::reduce_sum_i64(r->acc, src, r->extent, S.stream, &S.st.kernel_launches));
        k::PtrList dl{};
        for (int li = 0; li < S.V; ++li) dl.p[dl.n++] = r->dev[li];
        CUDA_TRY(k::apply_add_i64(dl, r->acc, r->extent, S.stream, &S.st.kernel_launches));
        TRY(dev_barrier());
        return 0;
    }
    k::PtrList src{};
    for (int li = 1; li < S.V; ++li) src.p[src.n++] = r->partial[li];
    CUDA_TRY(k::reduce_sum_i64(r->partial[0], src, r->extent, S.stream, &S.st.kernel_launches));
    if (S.use_nccl)
        NCCL_TRY(S.nccl->AllReduce(r->partial[0], r->partial[0], (size_t)r->extent, ncclInt64, ncclSum, S.comm, S.stream));
    k::PtrList dl{};
    for (int li = 0; li < S.V; ++li) dl.p[dl.n++] = r->dev[li];
    CUDA_TRY(k::apply_add_i64(dl, r->partial[0], r->extent, S.stream, &S.st.kernel_launches));
    return 0;
}

// Device-side precondition failures of bodies (d_flag[1]) surface at the next synchronising call.
int check_data_flag() {
    if (S.dry) return 0;
    TRY(flush_acct());
    CUDA_TRY(cudaMemcpyAsync(S.h_pin, S.d_flag, 3 * sizeof(int), cudaMemcpyDeviceToHost, S.stream));
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    const int* f = (const int*)S.h_pin;
    const int grid = f[1], scat = f[2];
    if (grid || scat) {
        CUDA_TRY(cudaMemsetAsync(S.d_flag + 1, 0, 2 * sizeof(int), S.stream));
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        if (grid)
            return fail(ACCMG_EDATA, "kmeans: a point is not on the 2^-shift fixed-point grid (|x*2^shift| < 2^31), "
                                     "or not finite in exact mode", false);
        return fail(ACCMG_EDATA, "scatter: an index lies in no partition's write window (negative, >= m, or a gap); "
                                 "its write was dropped", false);
    }
    return 0;
}

void free_region(accmg_region_s* r) {
    if (!S.dry) {
        cudaStreamSynchronize(S.stream);
        for (auto p : r->opened) cudaIpcCloseMemHandle(p);
        for (auto p : r->opened_partial) cudaIpcCloseMemHandle(p);
        r->opened.clear();
        r->opened_partial.clear();
        if (S.p2p) {  // nobody frees memory a peer may still have mapped
            std::string err;
            S.boot.barrier(&err);
        }
        if (r->vmm) free_vmm_region(r);
        for (int li = 0; li < (int)r->abase.size(); ++li)
            if (r->abase[li]) {
                const Ival& a = r->arange[first_local() + li];
                dfree(r->abase[li], (a.hi - a.lo) * r->esize, false);
            }
        for (auto& t : r->trk) {
            dfree(t.l1, t.nwords * 4, true);
            dfree(t.l2, t.nl2 * 4, true);
            dfree(t.tile_counts, t.ntiles * 24, true);
            dfree(t.tile_offs, t.ntiles * 24, true);
            dfree(t.tile_edges, t.ntiles * 8, true);
            dfree(t.totals, 64, true);
            dfree(t.packed, t.packed_cap, true);
            dfree(t.snap_l1, t.nwords * 4, true);
            dfree(t.snap_l2, t.nl2 * 4, true);
        }
        for (auto p : r->partial) dfree(p, r->extent * 8, true);
        dfree(r->acc, r->extent * 8, true);
    }
    delete r;
}

}  // namespace

// =================================================================================================
extern "C" {

int accmg_nccl_unique_id(uint8_t out[128]) {
    if (!out) return fail(ACCMG_EINVAL, "nccl_unique_id: null", false);
    const char* why = nullptr;
    accmg::NcclApi* n = accmg::nccl_api(&why);
    if (!n) return fail(ACCMG_ENCCL, why ? why : "NCCL unavailable", false);
    ncclUniqueId id;
    ncclResult_t r = n->GetUniqueId(&id);
    if (r != ncclSuccess) return fail(ACCMG_ENCCL, n->GetErrorString(r), false);
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    std::memcpy(out, &id, 128);
    return 0;
}

int accmg_init(const accmg_config* cfg) {
    if (S.init) return fail(ACCMG_ESTATE, "init: already initialised", false);
    if (!cfg) return fail(ACCMG_EINVAL, "init: null config", false);
    const accmg_config c = *cfg;
    if (c.world_size < 1 || c.rank < 0 || c.rank >= c.world_size) return fail(ACCMG_EINVAL, "init: bad world_size/rank", false);
    if (c.num_partitions < 1 || c.num_partitions % c.world_size != 0)
        return fail(ACCMG_EINVAL, "init: num_partitions must be a positive multiple of world_size", false);
    if (c.num_partitions > 64) return fail(ACCMG_EUNSUPPORTED, "init: at most 64 partitions", false);
    int64_t cb = c.dirty_chunk_bytes ? c.dirty_chunk_bytes : (1 << 20);
    if (cb < 256 || (cb & (cb - 1))) return fail(ACCMG_EINVAL, "init: dirty_chunk_bytes must be a power of two >= 256", false);
    if (c.exchange_mode != ACCMG_XCHG_AUTO && c.exchange_mode != ACCMG_XCHG_NCCL_ALL &&
        c.exchange_mode != ACCMG_XCHG_NCCL)
        return fail(ACCMG_EINVAL, "init: bad exchange_mode", false);
    S = State();
    S.cfg = c;
    S.P = c.num_partitions;
    S.W = c.world_size;
    S.rank = c.rank;
    S.V = S.P / S.W;
    S.dry = c.device < 0;
    S.nccl_all = c.exchange_mode == ACCMG_XCHG_NCCL_ALL;
    S.p2p = !S.dry && S.W > 1 && c.exchange_mode == ACCMG_XCHG_AUTO;
    S.use_nccl = !S.dry && (S.nccl_all || (S.W > 1 && c.exchange_mode == ACCMG_XCHG_NCCL));
    S.chunk_bytes = cb;
    if (c.dirty_protocol != ACCMG_DIRTY_RUNS && c.dirty_protocol != ACCMG_DIRTY_CHUNKS)
        return fail(ACCMG_EINVAL, "init: bad dirty_protocol", false);
    S.chunks = c.dirty_protocol == ACCMG_DIRTY_CHUNKS;
    if (c.halo_mode != ACCMG_HALO_AUTO && c.halo_mode != ACCMG_HALO_PULL)
        return fail(ACCMG_EINVAL, "init: bad halo_mode", false);
    if (c.multicast != ACCMG_MC_OFF && c.multicast != ACCMG_MC_AUTO && c.multicast != ACCMG_MC_VMM)
        return fail(ACCMG_EINVAL, "init: bad multicast", false);
    S.halo_pull = c.halo_mode == ACCMG_HALO_PULL;
    if (S.chunks && S.use_nccl) return fail(ACCMG_EUNSUPPORTED, "init: the chunk protocol needs a same-node transport", false);
    if (S.dry) {
        S.init = true;
        return 0;
    }
    CUDA_TRY(cudaSetDevice(c.device));
    CUDA_TRY(cudaStreamCreateWithFlags(&S.stream, cudaStreamNonBlocking));
    TRY(dmalloc((void**)&S.scratch, 2 * k::kScatterBlocks * 8, true));
    TRY(dmalloc((void**)&S.d_sizes, (size_t)4 * 8 * 16 * S.P * (S.W + 1), true));
    TRY(dmalloc((void**)&S.d_flag, 16, true));
    // [V] per-loop miss counters, [64) window starts at 2*64, ends at 3*64, running total at 4*64
    TRY(dmalloc((void**)&S.d_miss, sizeof(int64_t) * 5 * 64, true));
    S.d_miss_total = S.d_miss + 4 * 64;
    CUDA_TRY(cudaMemsetAsync(S.d_miss, 0, sizeof(int64_t) * 5 * 64, S.stream));
    CUDA_TRY(cudaHostAlloc((void**)&S.h_pin, (size_t)(kPinMiss + 128) * 8, cudaHostAllocDefault));
    CUDA_TRY(cudaHostAlloc((void**)&S.h_acct, (size_t)kAcctSlots * 4 * 8, cudaHostAllocDefault));
    CUDA_TRY(cudaMemsetAsync(S.d_flag, 0, 16, S.stream));
    if (S.p2p) {
        std::string err;
        if (!S.boot.open(c.nccl_unique_id, S.rank, S.W, &err)) return fail(ACCMG_ESTATE, err, true);
        TRY(dmalloc((void**)&S.sig, 8 * 64, true));
        CUDA_TRY(cudaMemset(S.sig, 0, 8 * 64));
        CUDA_TRY(cudaDeviceSynchronize());
        std::vector<void*> mine{S.sig};
        TRY(exchange_ptrs(mine, S.peer_sig, S.sig_opened));
        if (c.multicast == ACCMG_MC_AUTO && S.V == 1) {
            // the same answer on every rank of the node; a failure later still falls back per region
            S.mc_ok = accmg::vmm::mc_probe(S.W, 2u << 20, &S.mc_why) == 0;
        }
    }
    if (S.use_nccl) {
        const char* why = nullptr;
        S.nccl = accmg::nccl_api(&why);
        if (!S.nccl) return fail(ACCMG_ENCCL, why ? why : "NCCL unavailable", true);
        ncclUniqueId id;
        if (S.W == 1) NCCL_TRY(S.nccl->GetUniqueId(&id));
        else std::memcpy(&id, c.nccl_unique_id, 128);
        NCCL_TRY(S.nccl->CommInitRank(&S.comm, S.W, id, S.rank));
    }
    S.init = true;
    return 0;
}

int accmg_finalize(void) {
    if (!S.init) return fail(ACCMG_ESTATE, "finalize: not initialised", false);
    if (!S.dry) {
        cudaSetDevice(S.cfg.device);
        cudaStreamSynchronize(S.stream);
    }
    for (auto* r : S.regions) free_region(r);
    S.regions.clear();
    if (S.p2p) {
        for (auto p : S.sig_opened) cudaIpcCloseMemHandle(p);
        std::string err;
        S.boot.barrier(&err);
        dfree(S.sig, 0, true);
        S.boot.close();
    }
    if (!S.dry) {
        dfree(S.scratch, 0, true);
        dfree(S.d_sizes, 0, true);
        dfree(S.d_flag, 0, true);
        dfree(S.d_miss, 0, true);
        for (auto& D : S.deep)
            for (int q = 0; q < 2; ++q) dfree(D.alloc[q], (D.hi - D.lo) * 4, true);
        for (auto p : S.miss_recs) dfree(p, 0, true);
        dfree(S.recv, 0, true);
        cache_release();
        if (S.h_pin) cudaFreeHost(S.h_pin);
        if (S.h_acct) cudaFreeHost(S.h_acct);
        for (auto& p : S.prof) { cudaEventDestroy(p.a); cudaEventDestroy(p.b); }
        for (auto e : S.ev_free) cudaEventDestroy(e);
        if (S.comm) S.nccl->CommDestroy(S.comm);
        if (S.stream) cudaStreamDestroy(S.stream);
    }
    S = State();
    return 0;
}

int accmg_region_create(void* host_array, size_t elem_size, int64_t extent, accmg_region* out) {
    GUARD();
    NvtxScope nv("accmg_region_create");
    if (!host_array || !out || extent < 1) return fail(ACCMG_EINVAL, "region_create: null pointer or extent < 1", false);
    if (elem_size != 1 && elem_size != 2 && elem_size != 4 && elem_size != 8)
        return fail(ACCMG_EINVAL, "region_create: elem_size must be 1, 2, 4 or 8", false);
    auto* r = new accmg_region_s();
    r->id = S.next_id++;
    r->host = static_cast<uint8_t*>(host_array);
    r->esize = (int64_t)elem_size;
    r->extent = extent;
    r->valid.assign(S.P, IntervalSet());
    r->last_read.assign(S.P, IntervalSet());
    r->host_valid = IntervalSet(0, extent);
    r->trk.assign(S.V, Trk());
    r->dev.assign(S.V, nullptr);
    r->abase.assign(S.V, nullptr);
    r->arange.assign(S.P, Ival{0, 0});
    r->gdev.assign(S.P, nullptr);
    r->partial.assign(S.V, nullptr);
    // replicas are allocated on first use, sized to what each partition needs (ensure_alloc)
    S.regions.push_back(r);
    *out = r;
    return 0;
}

int accmg_region_destroy(accmg_region r) {
    GUARD();
    NvtxScope nv("accmg_region_destroy");
    auto it = std::find(S.regions.begin(), S.regions.end(), r);
    if (it == S.regions.end()) return fail(ACCMG_EINVAL, "region_destroy: unknown region", false);
    S.regions.erase(it);
    free_region(r);
    return 0;
}

namespace {
// One predicted-halo push: partition g's body also stores elements [lo, hi) of descriptor desc's
// array (rows of g's write window) into partition h's replica.
struct PushPiece {
    int desc, g, h;
    int64_t lo, hi;
};

// Plans the pushes of one loop and sets S.cur_push for the local partitions. Only bodies that can
// store their output rows twice take part (2-D Jacobi, output = descriptor 1). A piece is
// W_g ∩ last_read[h] ∩ valid[h]: rows g writes that h read in the last loop reading this array (so
// h is predicted to read them next, L125) and whose other elements h already holds (the body
// stores only the interior columns; the rest of the row is unchanged and must be valid there).
// Pieces must be whole rows, at most kMaxPush per writer, and the target replica must be
// addressable (same process, or P2P mappings). The plan is a pure function of the global state, so
// every process computes the same validity and byte counts.
int plan_pushes(int body_id, const accmg_access* descs, const void* args,
                const std::vector<std::vector<IntervalSet>>& need, std::vector<PushPiece>& out) {
    S.cur_push.assign(S.V, k::HaloPush{});
    if (S.halo_pull || S.P < 2 || body_id != ACCMG_BODY_JACOBI2D_5PT) return 0;
    const int di = 1;
    const accmg_access& d = descs[di];
    if (!d.declared) return 0;
    accmg_region_s* r = d.region;
    const int64_t cols = static_cast<const accmg_args_jacobi2d*>(args)->cols;
    for (int g = 0; g < S.P; ++g) {
        std::vector<PushPiece> mine;
        bool ok = true;
        for (int h = 0; h < S.P && ok; ++h) {
            if (h == g || r->last_read[h].empty()) continue;
            if (!(rank_of(h) == rank_of(g) || S.p2p)) continue;  // unreachable without a mapping
            IntervalSet piece = need[di][g].intersect(r->last_read[h]).intersect(r->valid[h]);
            for (auto& iv : piece.items()) {
                if (iv.lo % cols || iv.hi % cols || (int)mine.size() == k::kMaxPush) {
                    ok = false;
                    break;
                }
                mine.push_back({di, g, h, iv.lo, iv.hi});
            }
        }
        if (!ok || mine.empty()) continue;
        for (auto& pc : mine) {
            out.push_back(pc);
            const int64_t nb = (pc.hi - pc.lo) * r->esize;
            if (local(pc.h)) {  // bytes are counted by the receiving process (as for pulls)
                S.st.bytes_interpartition += nb;
                S.st.bytes_declared += nb;
                S.st.bytes_link += nb;
                if (rank_of(pc.g) != rank_of(pc.h)) {
                    S.st.bytes_remote += nb;
                    S.st.bytes_link_remote += nb;
                }
            }
            if (local(g) && !S.dry) {
                k::HaloPush& hp = S.cur_push[lidx(g)];
                uint8_t* base = S.p2p ? r->gdev[pc.h] : r->dev[lidx(pc.h)];
                hp.dst[hp.n] = reinterpret_cast<float*>(base);
                hp.lo[hp.n] = pc.lo / cols;
                hp.hi[hp.n] = pc.hi / cols;
                ++hp.n;
            }
        }
    }
    return 0;
}
}  // namespace

int accmg_loop_launch(const accmg_bounds* bounds, int body_id, const accmg_access* descs, int n_descs,
                      const void* args, size_t args_bytes) {
    GUARD();
    NvtxScope nv("accmg_loop_launch");
    if (!bounds || !descs || !args) return fail(ACCMG_EINVAL, "loop_launch: null argument", false);
    if (n_descs < 1 || n_descs > 16) return fail(ACCMG_EINVAL, "loop_launch: n_descs must be 1..16", false);
    BodySpec spec;
    if (!body_spec(body_id, &spec)) return fail(ACCMG_EINVAL, "loop_launch: unknown body_id", false);
    if (args_bytes != spec.args) return fail(ACCMG_EINVAL, "loop_launch: args_bytes does not match the body", false);
    if (bounds->ndim != spec.ndim) return fail(ACCMG_EINVAL, "loop_launch: wrong bounds.ndim for the body", false);
    for (int i = 0; i < bounds->ndim; ++i)
        if (bounds->hi[i] < bounds->lo[i]) return fail(ACCMG_EINVAL, "loop_launch: bounds hi < lo", false);
    if (n_descs != spec.n) return fail(ACCMG_EINVAL, "loop_launch: wrong number of descriptors for the body", false);
    for (int i = 0; i < n_descs; ++i) {
        const accmg_access& d = descs[i];
        if (std::find(S.regions.begin(), S.regions.end(), d.region) == S.regions.end())
            return fail(ACCMG_EINVAL, "loop_launch: descriptor " + std::to_string(i) + " has an unknown region", false);
        if (d.mode != spec.mode[i]) return fail(ACCMG_EINVAL, "loop_launch: descriptor " + std::to_string(i) + " has the wrong mode", false);
        if (d.region->esize != spec.esize[i])
            return fail(ACCMG_EINVAL, "loop_launch: descriptor " + std::to_string(i) + " has the wrong element size", false);
        if (d.declared && (d.stride <= 0 || d.left < 0 || d.right < 0))
            return fail(ACCMG_EINVAL, "loop_launch: declared window needs stride > 0, left/right >= 0", false);
        if (d.mode == ACCMG_REDUCE_SUM && d.declared)
            return fail(ACCMG_EINVAL, "loop_launch: REDUCE_SUM destinations are replicated (declared = 0)", false);
        for (int j = 0; j < i; ++j)
            if (descs[j].region == d.region) return fail(ACCMG_EINVAL, "loop_launch: a region appears twice", false);
    }
    TRY(validate_body(bounds, body_id, descs, args));

    // 1. task mapping (L108)
    std::vector<int64_t> ca(S.P), cb(S.P);
    for (int g = 0; g < S.P; ++g) chunk_of(bounds->lo[0], bounds->hi[0], S.P, g, &ca[g], &cb[g]);
    // 2. needs per descriptor: declared window (distribution) or whole array (replica)
    std::vector<std::vector<IntervalSet>> need(n_descs, std::vector<IntervalSet>(S.P));
    for (int i = 0; i < n_descs; ++i)
        for (int g = 0; g < S.P; ++g)
            need[i][g] = descs[i].declared ? window(descs[i], ca[g], cb[g], descs[i].region->extent)
                                           : IntervalSet(0, descs[i].region->extent);
    // owner computes: declared write windows must not overlap (G14)
    for (int i = 0; i < n_descs; ++i)
        if (descs[i].declared && (descs[i].mode & ACCMG_W))
            for (int g = 0; g < S.P; ++g)
                for (int h = 0; h < g; ++h)
                    if (need[i][g].overlaps(need[i][h]))
                        return fail(ACCMG_ECONFLICT, "declared write windows of two partitions overlap (G14)", false);
    // §8 f3: arrays written without a declared pattern get VMM replicas shared through descriptors
    // (and a multicast binding where available) at their first allocation
    if (S.p2p && S.V == 1 && S.cfg.multicast != ACCMG_MC_OFF)
        for (int i = 0; i < n_descs; ++i) {
            accmg_region_s* r = descs[i].region;
            bool fresh = !r->vmm;
            for (int g = 0; g < S.P && fresh; ++g) fresh = r->arange[g].hi <= r->arange[g].lo;
            if (fresh && (descs[i].mode & ACCMG_W) && descs[i].mode != ACCMG_REDUCE_SUM && !descs[i].declared &&
                (r->esize == 4 || r->esize == 8))
                TRY(setup_vmm_region(r));
        }
    // window-sized replicas: every partition's allocation covers what it needs (f4)
    for (int i = 0; i < n_descs; ++i) TRY(ensure_alloc(descs[i].region, need[i], descs[i].declared ? descs[i].stride : 0));
    // 3. data loader: plan all pulls from the pre-phase state, then run them
    std::vector<Xfer> xs;
    for (int i = 0; i < n_descs; ++i) plan_pulls(descs[i].region, need[i], xs);
    TRY(run_xfers(xs));
    // P2P: peers write into this process's replicas during the loop (the dirty-element pushes of
    // undeclared writes, the writing body's predicted halo pushes), so the loader's copies into
    // them (host copy-in, pulls) must have landed before any peer's body starts; without this a
    // fast peer's push of loop 0 could be overwritten by a slow rank's copy-in of the same rows.
    // The plan covers every partition, so every rank takes this branch (barrier epochs in step).
    if (S.p2p && !xs.empty()) TRY(dev_barrier());
    for (int i = 0; i < n_descs; ++i)
        for (int g = 0; g < S.P; ++g) descs[i].region->valid[g].add(need[i][g]);
    // predicted-halo push (halo_mode AUTO, L125: iterative codes reuse their access patterns)
    std::vector<PushPiece> pushes;
    TRY(plan_pushes(body_id, descs, args, need, pushes));

    std::vector<bool> tracked(n_descs, false);
    std::vector<accmg_region_s*> tracked_regs;
    for (int i = 0; i < n_descs; ++i)
        // with a single partition there is no other replica to keep coherent: no tracking
        // (kept under debug_checks so the artefacts can still be inspected)
        if ((descs[i].mode & ACCMG_W) && descs[i].mode != ACCMG_REDUCE_SUM && !descs[i].declared &&
            (S.P > 1 || S.cfg.debug_checks)) {
            tracked[i] = true;
            tracked_regs.push_back(descs[i].region);
        }
    if (!S.dry) {
        for (auto* r : tracked_regs)
            for (int li = 0; li < S.V; ++li) TRY(ensure_trk(r, li));
        for (int i = 0; i < n_descs; ++i)
            if (descs[i].mode == ACCMG_REDUCE_SUM) {
                accmg_region_s* r = descs[i].region;
                const bool fresh = !r->partial[0];
                for (int li = 0; li < S.V; ++li) {
                    if (!r->partial[li]) TRY(dmalloc((void**)&r->partial[li], r->extent * 8, true));
                    CUDA_TRY(cudaMemsetAsync(r->partial[li], 0, r->extent * 8, S.stream));
                }
                if (S.p2p && fresh) {  // same loop on every rank: publish the partials
                    TRY(dmalloc((void**)&r->acc, r->extent * 8, true));
                    std::vector<void*> mine(r->partial.begin(), r->partial.end()), all;
                    TRY(exchange_ptrs(mine, all, r->opened_partial));
                    r->gpartial.resize(S.P);
                    for (int g = 0; g < S.P; ++g) r->gpartial[g] = static_cast<int64_t*>(all[g]);
                }
            }
        if (body_id == ACCMG_BODY_SCATTER) {
            int64_t cap = 1;
            for (int g = 0; g < S.P; ++g) cap = std::max(cap, cb[g] - ca[g]);
            if (cap > S.miss_cap) {
                CUDA_TRY(cudaStreamSynchronize(S.stream));
                for (auto p : S.miss_recs) dfree(p, S.miss_cap * 8, true);
                S.miss_recs.assign(S.V, nullptr);
                for (int li = 0; li < S.V; ++li) TRY(dmalloc((void**)&S.miss_recs[li], cap * 8, true));  // 8-byte records
                S.miss_cap = cap;
            }
            CUDA_TRY(cudaMemsetAsync(S.d_miss, 0, sizeof(int64_t) * S.V, S.stream));
        }
        // 4. bodies on this process's partitions
        {
            ProfScope ps(0);
            for (int li = 0; li < S.V; ++li) {
                const int g = first_local() + li;
                if (cb[g] > ca[g]) TRY(launch_body(body_id, bounds, descs, args, g, ca[g], cb[g], tracked));
            }
        }
        // 5. coherence
        if (body_id == ACCMG_BODY_SCATTER) {
            // complete the buffered write misses in the owners' replicas (L137, L163): owner =
            // the partition whose declared write window holds the index
            ProfScope ps(2);
            accmg_region_s* r = descs[2].region;
            // window bounds staged through pinned memory: [0, 64) starts, [64, 128) ends
            int64_t* wb = S.h_pin + kPinMiss;
            int nb = 0;
            k::PtrList dl{};
            for (int g = 0; g < S.P; ++g) {
                IntervalSet w = window(descs[2], ca[g], cb[g], r->extent);
                if (w.empty()) continue;
                wb[nb] = w.items()[0].lo;
                wb[64 + nb] = w.items()[0].hi;
                ++nb;
                dl.p[dl.n++] = S.p2p ? (void*)r->gdev[g] : (void*)r->dev[lidx(g)];
            }
            CUDA_TRY(cudaMemcpyAsync(S.d_miss + 2 * 64, wb, sizeof(int64_t) * 128, cudaMemcpyHostToDevice, S.stream));
            for (int li = 0; li < S.V; ++li)
                CUDA_TRY(k::apply_misses(S.miss_recs[li], S.d_miss + li, S.miss_cap, dl, S.d_miss + 2 * 64,
                                         S.d_miss + 3 * 64, nb, S.d_miss_total, S.d_flag + 2, r->extent, S.stream,
                                         &S.st.kernel_launches));
        }
        if (!tracked_regs.empty()) TRY(propagate_dirty(tracked_regs));
        for (int i = 0; i < n_descs; ++i)
            if (descs[i].mode == ACCMG_REDUCE_SUM) TRY(merge_reduce(descs[i].region));
        // 6. global barrier (L64): no process starts the next loop before every peer finished
        // this one (its body, its pushes and its pulls from the others' replicas)
        TRY(dev_barrier());
    }
    for (int i = 0; i < n_descs; ++i) {
        accmg_region_s* r = descs[i].region;
        if (descs[i].mode == ACCMG_REDUCE_SUM) {
            // this process's V/P share of the ring all-reduce volume 2(P-1)*extent*8 (reading W8)
            const int64_t nb = 2 * (int64_t)(S.P - 1) * r->extent * 8 * S.V / S.P;
            S.st.bytes_reduce += nb;
            S.st.bytes_interpartition += nb;
            const int64_t sb = r->extent * 8;
            if (S.p2p) {  // every process reads the P-1 other partials (P-V of them remote)
                S.st.bytes_link += (int64_t)(S.P - 1) * sb;
                S.st.bytes_link_remote += (int64_t)(S.P - S.V) * sb;
            } else {      // local merge of V partials, then (NCCL) the ring all-reduce's share
                S.st.bytes_link += (int64_t)(S.V - 1) * sb;
                if (S.use_nccl && S.W > 1) {
                    const int64_t ring = 2 * (int64_t)(S.W - 1) * sb / S.W;
                    S.st.bytes_link += ring;
                    S.st.bytes_link_remote += ring;
                }
            }
            r->host_valid.clear();
        } else if (descs[i].mode & ACCMG_W) {
            if (descs[i].declared) {
                // the writer becomes the only holder of its write window, except for the rows it
                // pushed into its predicted readers' replicas
                for (int g = 0; g < S.P; ++g)
                    for (int h = 0; h < S.P; ++h)
                        if (h != g) r->valid[h].subtract(need[i][g]);
                for (auto& pc : pushes)
                    if (pc.desc == i) r->valid[pc.h].add(IntervalSet(pc.lo, pc.hi));
                for (int g = 0; g < S.P; ++g) r->host_valid.subtract(need[i][g]);
            } else {
                r->host_valid.clear();  // any element may have changed; every replica is coherent again
            }
        }
    }
    // remember this loop's declared read windows (the prediction of the next loop's reads)
    for (int i = 0; i < n_descs; ++i)
        if (descs[i].mode & ACCMG_R) {
            accmg_region_s* r = descs[i].region;
            for (int g = 0; g < S.P; ++g) r->last_read[g] = descs[i].declared ? need[i][g] : IntervalSet();
        }
    S.st.loops += 1;
    return 0;
}

static int sync_host_impl(accmg_region r, bool owned) {
    NvtxScope nv(owned ? "accmg_sync_to_host_owned" : "accmg_sync_to_host");
    GUARD();
    if (std::find(S.regions.begin(), S.regions.end(), r) == S.regions.end())
        return fail(ACCMG_EINVAL, "sync_to_host: unknown region", false);
    if (!owned && S.W > 1) {
        // make this process's first partition hold everything no local partition holds
        std::vector<IntervalSet> need(S.P);
        for (int q = 0; q < S.W; ++q) {
            IntervalSet held;
            for (int li = 0; li < S.V; ++li) held.add(r->valid[q * S.V + li]);
            IntervalSet m(0, r->extent);
            m.subtract(held);
            need[q * S.V].add(m);
            need[q * S.V].add(r->valid[q * S.V]);
        }
        TRY(ensure_alloc(r, need));
        std::vector<Xfer> xs;
        plan_pulls(r, need, xs);
        TRY(run_xfers(xs));
        for (int g = 0; g < S.P; ++g) r->valid[g].add(need[g]);
        TRY(dev_barrier());
    }
    TRY(check_data_flag());
    IntervalSet todo(0, r->extent);
    todo.subtract(r->host_valid);
    // full: copy each missing piece from the lowest-index local holder;
    // owned: only pieces whose lowest-index holder overall is local
    for (int g = 0; g < S.P && !todo.empty(); ++g) {
        if (!owned && !local(g)) continue;
        IntervalSet piece = todo.intersect(r->valid[g]);
        todo.subtract(piece);
        if (!local(g)) continue;
        for (auto& iv : piece.items()) {
            const int64_t off = iv.lo * r->esize, nb = (iv.hi - iv.lo) * r->esize;
            S.st.bytes_d2h += nb;
            if (!S.dry)
                CUDA_TRY(cudaMemcpyAsync(r->host + off, r->dev[lidx(g)] + off, (size_t)nb, cudaMemcpyDeviceToHost, S.stream));
            r->host_valid.add(iv.lo, iv.hi);
        }
    }
    if (!S.dry) CUDA_TRY(cudaStreamSynchronize(S.stream));
    if (!owned && !todo.empty()) return fail(ACCMG_ESTATE, "sync_to_host: range valid nowhere", false);
    return 0;
}

int accmg_sync_to_host(accmg_region r) { return sync_host_impl(r, false); }
int accmg_sync_to_host_owned(accmg_region r) { return sync_host_impl(r, true); }

int accmg_barrier(void) {
    GUARD();
    if (!S.dry) CUDA_TRY(cudaStreamSynchronize(S.stream));
    return check_data_flag();
}

int accmg_get_stats(accmg_stats* out) {
    GUARD();
    if (!out) return fail(ACCMG_EINVAL, "get_stats: null", false);
    if (!S.dry) {
        TRY(collect_prof());
        TRY(check_data_flag());
        CUDA_TRY(cudaMemcpyAsync(S.h_pin, S.d_miss_total, sizeof(int64_t), cudaMemcpyDeviceToHost, S.stream));
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        S.st.write_misses = S.h_pin[0] - S.miss_base;
        S.st.bytes_write_miss = S.st.write_misses * 12;  // int64 index + fp32 value delivered
    }
    *out = S.st;
    out->bytes_interpartition += out->bytes_write_miss;
    out->bytes_link += out->write_misses * 4;  // each completion stores the fp32 value in the owner's replica
    return 0;
}

int accmg_reset_stats(void) {
    GUARD();
    if (!S.dry) {
        TRY(collect_prof());
        // the miss counter is written on the library stream (non-blocking): read it there
        CUDA_TRY(cudaMemcpyAsync(S.h_pin, S.d_miss_total, sizeof(int64_t), cudaMemcpyDeviceToHost, S.stream));
        CUDA_TRY(cudaStreamSynchronize(S.stream));
        S.miss_base = S.h_pin[0];
    }
    const int64_t u = S.st.device_bytes_user, sy = S.st.device_bytes_system;
    S.st = accmg_stats{};
    S.st.device_bytes_user = u;
    S.st.device_bytes_system = sy;
    return 0;
}

int accmg_set_profile(int on) {
    GUARD();
    if (on != 0 && on != 1) return fail(ACCMG_EINVAL, "set_profile: 0 or 1", false);
    S.cfg.profile = on;
    return 0;
}

const char* accmg_last_error(void) { return S.err.c_str(); }

int accmg_multicast_probe(int num_devices, char* why, int cap) {
    if (num_devices < 1 || cap < 0) return fail(ACCMG_EINVAL, "multicast_probe: bad arguments", false);
    std::string w;
    int ok = 0;
    if (cudaFree(nullptr) != cudaSuccess) {  // context of the current device
        w = "no CUDA device";
    } else {
        ok = accmg::vmm::mc_probe(num_devices, 2u << 20, &w) == 0 ? 1 : 0;
    }
    if (why && cap > 0) {
        std::snprintf(why, (size_t)cap, "%s", ok ? "" : w.c_str());
    }
    return ok;
}

void* accmg_stream(void) { return S.init ? (void*)S.stream : nullptr; }

int accmg_chunk(int64_t lo, int64_t hi, int num_partitions, int partition, int64_t* a, int64_t* b) {
    if (!a || !b || num_partitions < 1 || partition < 0 || partition >= num_partitions || hi < lo)
        return fail(ACCMG_EINVAL, "chunk: bad arguments", false);
    chunk_of(lo, hi, num_partitions, partition, a, b);
    return 0;
}

static int debug_region(accmg_region r, int partition, Trk** t) {
    GUARD();
    if (S.dry) return fail(ACCMG_ESTATE, "debug: not available in dry-run mode", false);
    if (std::find(S.regions.begin(), S.regions.end(), r) == S.regions.end())
        return fail(ACCMG_EINVAL, "debug: unknown region", false);
    if (partition < 0 || partition >= S.P || !local(partition))
        return fail(ACCMG_EINVAL, "debug: partition does not live on this process", false);
    *t = &r->trk[lidx(partition)];
    return 0;
}

int accmg_debug_dirty_bitmap(accmg_region r, int partition, uint32_t* out_words, int64_t nwords) {
    Trk* t;
    TRY(debug_region(r, partition, &t));
    if (!t->has_snap) return fail(ACCMG_ESTATE, "debug: no bitmap snapshot (needs debug_checks=1 and an undeclared write)", false);
    if (!out_words || nwords != t->nwords) return fail(ACCMG_EINVAL, "debug: nwords must be ceil(extent/32)", false);
    CUDA_TRY(cudaMemcpyAsync(out_words, t->snap_l1, nwords * 4, cudaMemcpyDeviceToHost, S.stream));
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    return 0;
}

int accmg_debug_chunk_bits(accmg_region r, int partition, uint32_t* out_words, int64_t nwords) {
    Trk* t;
    TRY(debug_region(r, partition, &t));
    if (!t->has_snap) return fail(ACCMG_ESTATE, "debug: no bitmap snapshot (needs debug_checks=1 and an undeclared write)", false);
    if (!out_words || nwords != t->nl2) return fail(ACCMG_EINVAL, "debug: wrong chunk-bit word count", false);
    CUDA_TRY(cudaMemcpyAsync(out_words, t->snap_l2, nwords * 4, cudaMemcpyDeviceToHost, S.stream));
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    return 0;
}

int accmg_debug_packed(accmg_region r, int partition, void* out, int64_t cap, int64_t* used) {
    Trk* t;
    TRY(debug_region(r, partition, &t));
    if (!t->has_packed) return fail(ACCMG_ESTATE, "debug: no packed buffer yet", false);
    if (used) *used = t->packed_bytes;
    if (out && cap > 0) {
        CUDA_TRY(cudaMemcpyAsync(out, t->packed, (size_t)std::min(cap, t->packed_bytes), cudaMemcpyDeviceToHost, S.stream));
        CUDA_TRY(cudaStreamSynchronize(S.stream));
    }
    return 0;
}

int accmg_debug_replica(accmg_region r, int partition, void* out) {
    Trk* t;
    TRY(debug_region(r, partition, &t));
    if (!out) return fail(ACCMG_EINVAL, "debug: null", false);
    const Ival a = r->arange[partition];
    if (a.hi > a.lo)
        CUDA_TRY(cudaMemcpyAsync(static_cast<uint8_t*>(out) + a.lo * r->esize, r->dev[lidx(partition)] + a.lo * r->esize,
                                 (size_t)((a.hi - a.lo) * r->esize), cudaMemcpyDeviceToHost, S.stream));
    CUDA_TRY(cudaStreamSynchronize(S.stream));
    return 0;
}

int accmg_debug_valid(accmg_region r, int partition, int64_t* out_pairs, int64_t cap, int64_t* n) {
    if (S.sticky) return S.sticky;
    if (!S.init) return fail(ACCMG_ESTATE, "accmg: not initialised", false);
    if (std::find(S.regions.begin(), S.regions.end(), r) == S.regions.end())
        return fail(ACCMG_EINVAL, "debug: unknown region", false);
    if (partition < -1 || partition >= S.P) return fail(ACCMG_EINVAL, "debug: bad partition", false);
    const IntervalSet& v = partition < 0 ? r->host_valid : r->valid[partition];
    if (n) *n = (int64_t)v.items().size();
    for (int64_t i = 0; i < cap && i < (int64_t)v.items().size(); ++i) {
        out_pairs[2 * i] = v.items()[i].lo;
        out_pairs[2 * i + 1] = v.items()[i].hi;
    }
    return 0;
}

}  // extern "C"

extern "C" int accmg_unique_id(uint8_t out[128]) {
    if (!out) return fail(ACCMG_EINVAL, "unique_id: null", false);
    FILE* f = std::fopen("/dev/urandom", "rb");
    if (!f || std::fread(out, 1, 128, f) != 128) {
        if (f) std::fclose(f);
        return fail(ACCMG_ESTATE, "unique_id: cannot read /dev/urandom", false);
    }
    std::fclose(f);
    return 0;
}
