// Coherence of replicated arrays written without a declared pattern (paper L129-135 §IV.D.1;
// north star (4) and (5)).
//
// After the loop body set the two-level dirty bits, the sender compacts its dirty elements into
// the canonical packed buffer:
//   uint64 n_runs, uint64 n_elems, int64 run_start[n_runs], int64 run_end[n_runs] (exclusive),
//   payload = the values of the dirty elements, runs in ascending order;
// receivers scatter the runs back at the same global indices. Chunks whose second-level bit is
// clear are skipped without reading their first-level words ("the inter-GPU communication
// manager avoids unnecessary data transfers at the chunks which have no dirty data", L135).
//
// Passes: count (per 2048-word tile: run starts / run ends / elements, via the word masks
//   start = w & ~((w << 1) | msb(prev)),  end = w & ~((w >> 1) | (lsb(next) << 31))),
// scan (one block: tile offsets + header; clears L2), write (persistent producer/consumer kernel:
// bulk-copied bitmap words and values, block scans of word popcounts, coalesced payload stores;
// clears L1 as it goes). HBM-bound: per dirty element 1/8 B bitmap + esize read + esize written,
// + 16 B per run.
#include "kernels.h"
#include "tma_host.h"
#include "tma_dev.cuh"
#include "track.cuh"

namespace accmg {
namespace k {
namespace {

constexpr int kThreads = 256;
constexpr int kWordsPerThread = kTileWords / kThreads;  // 8

__device__ __forceinline__ uint32_t start_mask(uint32_t w, uint32_t prev) { return w & ~((w << 1) | (prev >> 31)); }
__device__ __forceinline__ uint32_t end_mask(uint32_t w, uint32_t next) { return w & ~((w >> 1) | (next << 31)); }

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(dev::kFull, v, o);
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T n = __shfl_up_sync(dev::kFull, v, o);
        if (lane >= o) v += n;
    }
    return v;
}

__global__ void __launch_bounds__(kThreads)
count_k(const uint32_t* __restrict__ l1, const uint32_t* __restrict__ l2, int64_t nwords, int cw_log2,
        int64_t* __restrict__ tile_counts, uint32_t* __restrict__ tile_edges) {
    const int64_t t = blockIdx.x;
    const int64_t w0 = t * kTileWords;
    const int64_t w1 = w0 + kTileWords < nwords ? w0 + kTileWords : nwords;
    __shared__ int dirty;
    __shared__ int64_t red[3][kThreads / 32];
    if (threadIdx.x == 0) dirty = 0;
    __syncthreads();
    for (int64_t c = (w0 >> cw_log2) + threadIdx.x; c <= ((w1 - 1) >> cw_log2); c += kThreads)
        if ((l2[c >> 5] >> (c & 31)) & 1u) dirty = 1;
    __syncthreads();
    if (!dirty) {
        if (threadIdx.x == 0) {
            tile_counts[3 * t] = tile_counts[3 * t + 1] = tile_counts[3 * t + 2] = 0;
            tile_edges[2 * t] = tile_edges[2 * t + 1] = 0u;
        }
        return;
    }
    int64_t ns = 0, ne = 0, nel = 0;
    const int64_t ws = w0 + (int64_t)threadIdx.x * kWordsPerThread;
    if (ws + kWordsPerThread <= w1 && (reinterpret_cast<uintptr_t>(l1 + ws) & 15) == 0) {
        // full group: two 128-bit loads (coalesced across the warp) and the two neighbour words
        static_assert(kWordsPerThread == 8, "two uint4 per thread");
        const uint4 a = *reinterpret_cast<const uint4*>(l1 + ws);
        const uint4 b = *reinterpret_cast<const uint4*>(l1 + ws + 4);
        const uint32_t wv[10] = {ws >= 1 ? l1[ws - 1] : 0u, a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w,
                                 ws + 8 < nwords ? l1[ws + 8] : 0u};
#pragma unroll
        for (int j = 1; j <= 8; ++j) {
            ns += __popc(start_mask(wv[j], wv[j - 1]));
            ne += __popc(end_mask(wv[j], wv[j + 1]));
            nel += __popc(wv[j]);
        }
    } else if (ws < w1) {
        uint32_t prev = ws >= 1 ? l1[ws - 1] : 0u;  // count pass clears nothing: neighbours are stable
        uint32_t cur = l1[ws];
#pragma unroll
        for (int j = 0; j < kWordsPerThread; ++j) {
            const int64_t w = ws + j;
            if (w >= w1) break;
            const uint32_t next = (w + 1 < nwords) ? l1[w + 1] : 0u;
            ns += __popc(start_mask(cur, prev));
            ne += __popc(end_mask(cur, next));
            nel += __popc(cur);
            prev = cur;
            cur = next;
        }
    }
    ns = warp_sum(ns); ne = warp_sum(ne); nel = warp_sum(nel);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) { red[0][warp] = ns; red[1][warp] = ne; red[2][warp] = nel; }
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t a = 0, b = 0, c = 0;
        for (int i = 0; i < kThreads / 32; ++i) { a += red[0][i]; b += red[1][i]; c += red[2][i]; }
        tile_counts[3 * t] = a; tile_counts[3 * t + 1] = b; tile_counts[3 * t + 2] = c;
        tile_edges[2 * t] = l1[w0];
        tile_edges[2 * t + 1] = l1[w1 - 1];
    }
}

// One block: exclusive scan of the per-tile triples {starts, ends, elems}, 1024 tiles per step
// (coalesced loads of the next step issued before the current one is scanned; warp-shuffle scans;
// double-buffered warp totals, so two barriers per step and every thread carries the running
// totals in registers), then the L2 popcount + clear.
__global__ void __launch_bounds__(1024)
scan_k(const int64_t* __restrict__ tile_counts, int64_t ntiles, int64_t* __restrict__ tile_offs,
       int64_t* __restrict__ totals, uint32_t* __restrict__ l2, int64_t nl2words) {
    __shared__ int64_t wsum[2][3][32];
    __shared__ int64_t wtot[2][3];
    __shared__ unsigned long long nchunks;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) nchunks = 0ull;
    int64_t carry[3] = {0, 0, 0}, vn[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) vn[q] = tid < ntiles ? tile_counts[3 * tid + q] : 0;
    int buf = 0;
    for (int64_t base = 0; base < ntiles; base += 1024, buf ^= 1) {
        const int64_t t = base + tid, tn = t + 1024;
        int64_t v[3], inc[3];
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            v[q] = vn[q];
            vn[q] = tn < ntiles ? tile_counts[3 * tn + q] : 0;  // next step's loads in flight
            inc[q] = warp_incl_scan(v[q]);
            if (lane == 31) wsum[buf][q][warp] = inc[q];
        }
        __syncthreads();
        if (warp == 0) {
#pragma unroll
            for (int q = 0; q < 3; ++q) {
                const int64_t x = wsum[buf][q][lane];
                const int64_t xi = warp_incl_scan(x);
                wsum[buf][q][lane] = xi - x;  // exclusive warp offsets
                if (lane == 31) wtot[buf][q] = xi;
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            if (t < ntiles) tile_offs[3 * t + q] = carry[q] + wsum[buf][q][warp] + inc[q] - v[q];
            carry[q] += wtot[buf][q];
        }
    }
    unsigned long long pc = 0;
    for (int64_t w = tid; w < nl2words; w += 1024) { pc += __popc(l2[w]); l2[w] = 0u; }
    pc = warp_sum(pc);
    if (lane == 0) atomicAdd(&nchunks, pc);
    __syncthreads();
    if (tid == 0) {
        totals[0] = carry[0]; totals[1] = carry[2]; totals[2] = (int64_t)nchunks; totals[3] = carry[1];
    }
}

// Pass 3: persistent, warp-specialised.
// Measured: a one-tile-per-block kernel spends most of a tile's life in dependent global loads
// (tile counts -> bitmap words -> offsets, ~5 us each under full HBM load) before any payload
// moves, so it capped at ~4 TB/s whatever the ring depth. Here each block walks its tiles
// t = blockIdx.x + k * gridDim.x with one producer warp running ahead of eight consumer warps:
//  * producer (warp 8, one lane): reads the tile's counts / offsets / edge words into a
//    double-buffered tile record, bulk-copies (cp.async.bulk) the tile's 8 KiB of bitmap words
//    into that record and, for dense tiles, the values through an NST-stage ring of 8 KiB stages
//    (mbarrier full/empty pairs), skipping clean tiles; it is up to two tiles ahead;
//  * consumers (warps 0-7): per tile, clear the L1 words, scan the word popcounts (payload offset
//    of each word inside the tile), write the run starts / ends, then store the dirty elements of
//    each ring stage with coalesced stores (dense tiles) or gather them with kU predicated
//    coalesced loads in flight per warp (sparse / ragged / unaligned tiles).
constexpr int kU = 16;
constexpr int kPad = 4;  // sw[kPad - 1] = previous tile's last word; sw[kPad + nw] = next tile's first
constexpr uint32_t kStageBytes = 8192;
constexpr int64_t kDenseElems = (int64_t)kTileWords * 32 / 2;
constexpr int kConsumers = 256;  // warps 0-7; warp 8 is the producer

__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     dev::smem_u32(dst)),
                 "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(dev::smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory"); }

struct TileRec {  // one dirty tile, written by the producer before it arrives on the record's full barrier
    int64_t t, off_s, off_e, off_el;
    uint32_t edge_prev, edge_next;
    int nw, dense;  // t < 0: end of this block's tiles
};

// A push store: into one replica, or (push.mc) through the multicast address into all of them.
template <typename T>
__device__ __forceinline__ void push_store(const PtrList& push, int d, int64_t e, T v) {
    T* p = static_cast<T*>(push.p[d]) + e;
    if constexpr (sizeof(T) == 4) {
        if (push.mc) {
            asm volatile("multimem.st.relaxed.sys.global.b32 [%0], %1;" ::"l"(p), "r"(*reinterpret_cast<uint32_t*>(&v))
                         : "memory");
            return;
        }
    } else if constexpr (sizeof(T) == 8) {
        if (push.mc) {
            asm volatile("multimem.st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p),
                         "l"(*reinterpret_cast<unsigned long long*>(&v))
                         : "memory");
            return;
        }
    }
    *p = v;
}

template <typename T, int NST>
__global__ void __launch_bounds__(kConsumers + 32)
write_pipe_k(uint32_t* __restrict__ l1, int64_t nwords, int64_t extent, const int64_t* __restrict__ tile_counts,
             const int64_t* __restrict__ tile_offs, const uint32_t* __restrict__ tile_edges, int64_t ntiles,
             const T* __restrict__ values, uint8_t* __restrict__ packed, int64_t n_runs, int aligned,
             const PtrList push, int keep) {
    constexpr int SCW = kStageBytes / (32 * sizeof(T));  // words per stage
    constexpr int NSC = kTileWords / SCW;                 // stages per tile
    extern __shared__ __align__(128) unsigned char ring[];  // NST x kStageBytes
    __shared__ __align__(16) uint32_t sw[2][kTileWords + 2 * kPad];
    __shared__ int32_t spre[kTileWords];
    __shared__ int32_t wred[3][kConsumers / 32];
    __shared__ TileRec rec[2];
    __shared__ __align__(8) uint64_t full[NST], empty[NST], rfull[2], rempty[2];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int q = 0; q < NST; ++q) { dev::mbar_init(&full[q], 1); dev::mbar_init(&empty[q], kConsumers / 32); }
        for (int q = 0; q < 2; ++q) { dev::mbar_init(&rfull[q], 1); dev::mbar_init(&rempty[q], kConsumers / 32); }
        dev::mbar_fence_init();
    }
    __syncthreads();

    if (warp == kConsumers / 32) {  // ---------------- producer ----------------
        if (lane != 0) return;
        uint32_t seq = 0, kk = 0;
        for (int64_t t = blockIdx.x;; t += gridDim.x) {
            const bool end = t >= ntiles;
            const int64_t el = end ? 0 : tile_counts[3 * t + 2];
            if (!end && el == 0) continue;  // clean tile: nothing to pack
            const int b = kk & 1;
            dev::mbar_wait(&rempty[b], ((kk >> 1) & 1) ^ 1);  // consumers released this record
            TileRec& r = rec[b];
            if (end) {
                r.t = -1;
                dev::mbar_arrive(&rfull[b]);
                return;
            }
            const int64_t w0 = t * kTileWords;
            const int nw = (int)((w0 + kTileWords < nwords ? w0 + kTileWords : nwords) - w0);
            const bool dense = aligned && el >= kDenseElems && nw == kTileWords && (w0 + kTileWords) * 32 <= extent;
            r.t = t;
            r.off_s = tile_offs[3 * t];
            r.off_e = tile_offs[3 * t + 1];
            r.off_el = tile_offs[3 * t + 2];
            r.edge_prev = t > 0 ? tile_edges[2 * (t - 1) + 1] : 0u;
            r.edge_next = t + 1 < ntiles ? tile_edges[2 * (t + 1)] : 0u;
            r.nw = nw;
            r.dense = dense;
            if (nw == kTileWords) {  // the words are 16-byte aligned (w0 * 4 is a multiple of 8 KiB)
                dev::mbar_expect_tx(&rfull[b], kTileWords * 4);
                bulk_load(&sw[b][kPad], l1 + w0, kTileWords * 4, &rfull[b]);
            } else {
                dev::mbar_arrive(&rfull[b]);  // ragged last tile: the consumers load its words
            }
            ++kk;
            if (!dense) continue;
            for (int q = 0; q < NSC; ++q, ++seq) {
                const int st = seq % NST;
                dev::mbar_wait(&empty[st], ((seq / NST) & 1) ^ 1);
                dev::mbar_expect_tx(&full[st], kStageBytes);
                bulk_load(ring + st * kStageBytes, values + (w0 + (int64_t)q * SCW) * 32, kStageBytes, &full[st]);
            }
        }
    }

    // ---------------- consumers ----------------
    int64_t* run_start = reinterpret_cast<int64_t*>(packed + 16);
    int64_t* run_end = run_start + n_runs;
    T* payload = reinterpret_cast<T*>(packed + 16 + 16 * n_runs);
    const uint32_t lt = (1u << lane) - 1u;
    uint32_t seq = 0;
    for (uint32_t kk = 0;; ++kk) {
        const int b = kk & 1;
        dev::mbar_wait(&rfull[b], (kk >> 1) & 1);
        const TileRec r = rec[b];
        if (r.t < 0) break;
        uint32_t* W = sw[b];
        const int64_t w0 = r.t * kTileWords;
        const int nw = r.nw;
        if (nw == kTileWords) {
            uint4* g = reinterpret_cast<uint4*>(l1 + w0);
            for (int i = tid; i < kTileWords / 4; i += kConsumers) g[i] = make_uint4(0u, 0u, 0u, 0u);
        } else {
            for (int i = tid; i < nw; i += kConsumers) {
                W[kPad + i] = l1[w0 + i];
                l1[w0 + i] = 0u;
            }
        }
        if (tid == 0) {
            W[kPad - 1] = r.edge_prev;
            W[kPad + nw] = r.edge_next;
        }
        consumers_sync();
        // thread tid owns words [8 tid, 8 tid + 8): counts, then a block exclusive scan
        const int i0 = tid * kWordsPerThread;
        int cel = 0, cs = 0, ce = 0;
#pragma unroll
        for (int j = 0; j < kWordsPerThread; ++j) {
            const int i = i0 + j;
            if (i < nw) {
                const uint32_t w = W[kPad + i];
                cel += __popc(w);
                cs += __popc(start_mask(w, W[kPad + i - 1]));
                ce += __popc(end_mask(w, W[kPad + i + 1]));
            }
        }
        const int iel = warp_incl_scan(cel), is = warp_incl_scan(cs), ie = warp_incl_scan(ce);
        if (lane == 31) { wred[0][warp] = iel; wred[1][warp] = is; wred[2][warp] = ie; }
        consumers_sync();
        int oel = iel - cel, os = is - cs, oe = ie - ce;
        for (int i = 0; i < warp; ++i) { oel += wred[0][i]; os += wred[1][i]; oe += wred[2][i]; }
        {
            int64_t ks = r.off_s + os, ke = r.off_e + oe;
            int run = oel;
#pragma unroll
            for (int j = 0; j < kWordsPerThread; ++j) {
                const int i = i0 + j;
                if (i < nw) {
                    const uint32_t w = W[kPad + i];
                    spre[i] = run;
                    run += __popc(w);
                    const int64_t gw = w0 + i;
                    if (keep) {
                        for (uint32_t m = start_mask(w, W[kPad + i - 1]); m; m &= m - 1) run_start[ks++] = gw * 32 + (__ffs(m) - 1);
                        for (uint32_t m = end_mask(w, W[kPad + i + 1]); m; m &= m - 1) run_end[ke++] = gw * 32 + __ffs(m);
                    }
                }
            }
        }
        consumers_sync();
        T* tile_payload = payload + r.off_el;
        // the push-only case (nothing packed): replica by replica, a per-tile base pointer and
        // 32-bit offsets instead of a 64-bit global index and a pointer-list loop per element (the
        // stage is re-read from shared memory for each replica)
        if (r.dense && !keep && push.n >= 1) {
            for (int q = 0; q < NSC; ++q, ++seq) {
                const int st = seq % NST;
                dev::mbar_wait(&full[st], (seq / NST) & 1);
                const T* V = reinterpret_cast<const T*>(ring + st * kStageBytes);
                if (push.mc) {  // one store per dirty element, to every replica at once
#pragma unroll
                    for (int j = warp; j < SCW; j += kConsumers / 32) {
                        const int i = q * SCW + j;
                        if ((W[kPad + i] >> lane) & 1u) push_store(push, 0, (w0 + i) * 32 + lane, V[j * 32 + lane]);
                    }
                } else {
                    for (int d = 0; d < push.n; ++d) {
                        T* const pd = static_cast<T*>(push.p[d]) + w0 * 32;
#pragma unroll
                        for (int j = warp; j < SCW; j += kConsumers / 32) {
                            const int i = q * SCW + j;
                            if ((W[kPad + i] >> lane) & 1u) pd[i * 32 + lane] = V[j * 32 + lane];
                        }
                    }
                }
                __syncwarp();
                if (lane == 0) dev::mbar_arrive(&empty[st]);
            }
        } else if (r.dense) {
            for (int q = 0; q < NSC; ++q, ++seq) {
                const int st = seq % NST;
                dev::mbar_wait(&full[st], (seq / NST) & 1);
                const T* V = reinterpret_cast<const T*>(ring + st * kStageBytes);
#pragma unroll
                for (int j = warp; j < SCW; j += kConsumers / 32) {
                    const int i = q * SCW + j;
                    const uint32_t m = W[kPad + i];
                    if ((m >> lane) & 1u) {
                        const T v = V[j * 32 + lane];
                        if (keep) tile_payload[spre[i] + __popc(m & lt)] = v;
                        const int64_t e = (w0 + i) * 32 + lane;
                        for (int d = 0; d < push.n; ++d) push_store(push, d, e, v);
                    }
                }
                __syncwarp();
                if (lane == 0) dev::mbar_arrive(&empty[st]);
            }
        } else {
            const T* vt = values + w0 * 32 + lane;
            for (int base = warp * kU; base < nw; base += (kConsumers / 32) * kU) {
                uint32_t m[kU];
                T v[kU];
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    m[u] = base + u < nw ? W[kPad + base + u] : 0u;
                    v[u] = ((m[u] >> lane) & 1u) ? vt[(int64_t)(base + u) * 32] : T(0);
                }
#pragma unroll
                for (int u = 0; u < kU; ++u)
                    if ((m[u] >> lane) & 1u) {
                        if (keep) tile_payload[spre[base + u] + __popc(m[u] & lt)] = v[u];
                        const int64_t e = (w0 + base + u) * 32 + lane;
                        for (int d = 0; d < push.n; ++d) push_store(push, d, e, v[u]);
                    }
            }
        }
        consumers_sync();  // spre / wred / this record are free again
        if (lane == 0) dev::mbar_arrive(&rempty[b]);
    }
}

template <typename T, int NST>
cudaError_t launch_write_pipe_st(uint32_t* l1, int64_t nwords, int64_t extent, int64_t ntiles, const int64_t* tile_counts,
                                 const int64_t* tile_offs, const uint32_t* tile_edges, const void* values,
                                 uint8_t* packed, int64_t n_runs, const PtrList& push, cudaStream_t s, int keep) {
    auto kern = write_pipe_k<T, NST>;
    const size_t smem = (size_t)NST * kStageBytes;
    int per_sm = 1;
    cudaError_t e = kernel_prep(kern, kConsumers + 32, smem, &per_sm);
    if (e != cudaSuccess) return e;
    const int aligned = (reinterpret_cast<uintptr_t>(values) % 16) == 0;
    const int sms = sm_count_cached();
    int64_t grid = (int64_t)sms * (per_sm > 0 ? per_sm : 1);
    if (grid > ntiles) grid = ntiles;
    kern<<<(unsigned)grid, kConsumers + 32, smem, s>>>(l1, nwords, extent, tile_counts, tile_offs, tile_edges, ntiles,
                                                        static_cast<const T*>(values), packed, n_runs, aligned, push, keep);
    return cudaGetLastError();
}

// Ring depth 3 (4 blocks per SM). Measured (C5, P = 2 and 8, profiles/r01/compact_pipe.log): more
// blocks per SM beat deeper rings -- 3 stages 1.59 ms per loop, 6: 1.71, 10: 1.71, 24 (1 block per
// SM): 2.09; a one-tile-per-block kernel was 2.37 and a ballot-group write pass 2.21.
template <typename T>
cudaError_t launch_write_stream(uint32_t* l1, int64_t nwords, int64_t extent, int64_t ntiles, const int64_t* tile_counts,
                                const int64_t* tile_offs, const uint32_t* tile_edges, const void* values,
                                uint8_t* packed, int64_t n_runs, const PtrList& push, cudaStream_t s, int keep) {
    return launch_write_pipe_st<T, 3>(l1, nwords, extent, ntiles, tile_counts, tile_offs, tile_edges, values, packed,
                                      n_runs, push, s, keep);
}

// ---- scatter of packed runs ----------------------------------------------------------------------
__device__ __forceinline__ void seg(int64_t n, int b, int64_t& lo, int64_t& hi) {
    lo = n * b / kScatterBlocks;
    hi = n * (b + 1) / kScatterBlocks;
}

__global__ void __launch_bounds__(kThreads)
runlen_sum_k(const uint8_t* __restrict__ packed, int64_t n_runs, int64_t* __restrict__ scratch) {
    const int64_t* rs = reinterpret_cast<const int64_t*>(packed + 16);
    const int64_t* re = rs + n_runs;
    int64_t lo, hi;
    seg(n_runs, blockIdx.x, lo, hi);
    int64_t s = 0;
    for (int64_t r = lo + threadIdx.x; r < hi; r += kThreads) s += re[r] - rs[r];
    s = warp_sum(s);
    __shared__ int64_t red[kThreads / 32];
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t a = 0;
        for (int i = 0; i < kThreads / 32; ++i) a += red[i];
        scratch[blockIdx.x] = a;
    }
}

// Exclusive scan of the kScatterBlocks segment sums (one block; was a single-thread loop: 20 us).
__global__ void __launch_bounds__(1024) runlen_scan_k(int64_t* __restrict__ scratch) {
    static_assert(kScatterBlocks <= 1024, "one element per thread");
    __shared__ int64_t wsum[32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t v = tid < kScatterBlocks ? scratch[tid] : 0;
    const int64_t inc = warp_incl_scan(v);
    if (lane == 31) wsum[warp] = inc;
    __syncthreads();
    if (warp == 0) {
        const int64_t x = wsum[lane];
        wsum[lane] = warp_incl_scan(x) - x;
    }
    __syncthreads();
    if (tid < kScatterBlocks) scratch[kScatterBlocks + tid] = wsum[warp] + inc - v;
}

constexpr int kSU = 16;  // loads in flight per lane (scatter)

template <typename T>
__global__ void __launch_bounds__(kThreads)
scatter_k(const uint8_t* __restrict__ packed, int64_t n_runs, const PtrList dsts,
          const int64_t* __restrict__ scratch) {
    const int64_t* rs = reinterpret_cast<const int64_t*>(packed + 16);
    const int64_t* re = rs + n_runs;
    const T* payload = reinterpret_cast<const T*>(packed + 16 + 16 * n_runs);
    int64_t lo, hi;
    seg(n_runs, blockIdx.x, lo, hi);
    __shared__ int64_t s_start[kThreads], s_len[kThreads], s_off[kThreads];
    __shared__ int64_t carry, s_tot;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) carry = scratch[kScatterBlocks + blockIdx.x];
    __syncthreads();
    for (int64_t base = lo; base < hi; base += kThreads) {
        const int64_t r = base + tid;
        const int64_t len = r < hi ? re[r] - rs[r] : 0;
        // block exclusive scan of len
        int64_t inc = warp_incl_scan(len);
        __shared__ int64_t wsum[kThreads / 32];
        if (lane == 31) wsum[warp] = inc;
        __syncthreads();
        int64_t wo = 0;
        for (int i = 0; i < warp; ++i) wo += wsum[i];
        s_start[tid] = r < hi ? rs[r] : 0;
        s_len[tid] = len;
        s_off[tid] = carry + wo + inc - len;
        if (tid == kThreads - 1) s_tot = wo + inc;
        __syncthreads();
        if (tid == kThreads - 1) carry += wo + inc;
        const int nr = (int)((hi - base) < kThreads ? (hi - base) : kThreads);
        // the chunk's payload [p0, p0 + tot) split evenly over the warps (runs differ in length:
        // one run per warp left warps idle), each warp walking the runs that overlap its range
        const int64_t p0 = s_off[0], tot = s_tot;
        const int64_t plo = p0 + tot * warp / (kThreads / 32), phi = p0 + tot * (warp + 1) / (kThreads / 32);
        int q = 0;
        {
            int a = 0, b = nr - 1;  // first run q with s_off[q] + s_len[q] > plo
            while (a < b) {
                const int m = (a + b) >> 1;
                if (s_off[m] + s_len[m] > plo) b = m;
                else a = m + 1;
            }
            q = a;
        }
        for (; q < nr && s_off[q] < phi; ++q) {
            const int64_t st = s_start[q], of = s_off[q];
            const int64_t xa = (plo > of ? plo : of) - of, xb = (phi < of + s_len[q] ? phi : of + s_len[q]) - of;
            // kSU independent loads per lane in flight, then the stores to every destination
            for (int64_t x0 = xa; x0 < xb; x0 += 32 * kSU) {
                T v[kSU];
#pragma unroll
                for (int u = 0; u < kSU; ++u) {
                    const int64_t x = x0 + 32 * u + lane;
                    v[u] = x < xb ? payload[of + x] : T(0);
                }
                for (int d = 0; d < dsts.n; ++d) {
                    T* dp = static_cast<T*>(dsts.p[d]) + st;
#pragma unroll
                    for (int u = 0; u < kSU; ++u) {
                        const int64_t x = x0 + 32 * u + lane;
                        if (x < xb) dp[x] = v[u];
                    }
                }
            }
        }
        __syncthreads();
    }
}

// The paper's protocol (L133-135): for every chunk whose second-level bit is set, the whole chunk's
// first-level bits decide which elements overwrite the peers' copies ("merged by the dirty bits").
// One block per dirty chunk (grid-stride); each warp takes kMU consecutive words at a time: all
// their bitmap words, then all their dirty values are loaded (kMU x 128 B in flight per warp)
// before the stores to every destination; clears the chunk's L1 words afterwards.
constexpr int kMU = 8;
template <typename T>
__global__ void __launch_bounds__(kThreads)
chunk_merge_k(uint32_t* __restrict__ l1, const uint32_t* __restrict__ l2, int64_t nwords, int cw_log2,
              const T* __restrict__ src, const PtrList dsts) {
    const int64_t cwords = (int64_t)1 << cw_log2;
    const int64_t nchunks = (nwords + cwords - 1) / cwords;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int64_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
        if (!((l2[c >> 5] >> (c & 31)) & 1u)) continue;  // clean chunk: skipped (block-uniform)
        const int64_t w0 = c * cwords, w1 = w0 + cwords < nwords ? w0 + cwords : nwords;
        for (int64_t wb = w0 + (int64_t)warp * kMU; wb < w1; wb += (int64_t)(kThreads / 32) * kMU) {
            uint32_t m[kMU];
            T v[kMU];
#pragma unroll
            for (int u = 0; u < kMU; ++u) m[u] = wb + u < w1 ? l1[wb + u] : 0u;
#pragma unroll
            for (int u = 0; u < kMU; ++u) v[u] = ((m[u] >> lane) & 1u) ? src[(wb + u) * 32 + lane] : T(0);
            for (int d = 0; d < dsts.n; ++d) {
                T* dp = static_cast<T*>(dsts.p[d]);
#pragma unroll
                for (int u = 0; u < kMU; ++u)
                    if ((m[u] >> lane) & 1u) dp[(wb + u) * 32 + lane] = v[u];
            }
        }
        __syncthreads();
        for (int64_t w = w0 + threadIdx.x; w < w1; w += kThreads) l1[w] = 0u;
        __syncthreads();
    }
}

__global__ void reduce_sum_k(int64_t* __restrict__ acc, const PtrList srcs, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = acc[i];
        for (int j = 0; j < srcs.n; ++j) a += static_cast<const int64_t*>(srcs.p[j])[i];
        acc[i] = a;
    }
}

__global__ void apply_add_k(const PtrList dsts, const int64_t* __restrict__ acc, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = acc[i];
        for (int j = 0; j < dsts.n; ++j) static_cast<int64_t*>(dsts.p[j])[i] += a;
    }
}

__global__ void overlap_k(const uint32_t* __restrict__ a, const uint32_t* __restrict__ b, int64_t n, int* flag) {
    uint32_t acc = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        acc |= a[i] & b[i];
    if (__syncthreads_or(acc != 0u) && threadIdx.x == 0) atomicOr(flag, 1);
}

unsigned gs_blocks(int64_t n) {
    int64_t b = (n + 255) / 256;
    return (unsigned)(b < 148 * 8 ? (b < 1 ? 1 : b) : 148 * 8);
}

}  // namespace

cudaError_t compact_count(const uint32_t* l1, const uint32_t* l2, int64_t nwords, int chunk_words_log2,
                          int64_t ntiles, int64_t* tile_counts, uint32_t* tile_edges, cudaStream_t s,
                          int64_t* launches) {
    count_k<<<(unsigned)ntiles, kThreads, 0, s>>>(l1, l2, nwords, chunk_words_log2, tile_counts, tile_edges);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t compact_scan(const int64_t* tile_counts, int64_t ntiles, int64_t* tile_offs, int64_t* totals,
                         uint32_t* l2, int64_t nl2words, cudaStream_t s, int64_t* launches) {
    scan_k<<<1, 1024, 0, s>>>(tile_counts, ntiles, tile_offs, totals, l2, nl2words);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t compact_write(uint32_t* l1, int64_t nwords, int64_t extent, int64_t ntiles, const int64_t* tile_counts,
                          const int64_t* tile_offs, const uint32_t* tile_edges, const void* values,
                          int esize, uint8_t* packed, int64_t n_runs, const PtrList& push, cudaStream_t s,
                          int64_t* launches, int keep) {
    cudaError_t e;
    switch (esize) {
        case 1: e = launch_write_stream<uint8_t>(l1, nwords, extent, ntiles, tile_counts, tile_offs, tile_edges, values, packed, n_runs, push, s, keep); break;
        case 2: e = launch_write_stream<uint16_t>(l1, nwords, extent, ntiles, tile_counts, tile_offs, tile_edges, values, packed, n_runs, push, s, keep); break;
        case 4: e = launch_write_stream<uint32_t>(l1, nwords, extent, ntiles, tile_counts, tile_offs, tile_edges, values, packed, n_runs, push, s, keep); break;
        case 8: e = launch_write_stream<uint64_t>(l1, nwords, extent, ntiles, tile_counts, tile_offs, tile_edges, values, packed, n_runs, push, s, keep); break;
        default: return cudaErrorInvalidValue;
    }
    if (launches) *launches += 1;
    return e;
}

cudaError_t scatter_packed(const uint8_t* packed, int64_t n_runs, const PtrList& dsts, int esize,
                           int64_t* scratch, cudaStream_t s, int64_t* launches) {
    if (n_runs == 0 || dsts.n == 0) return cudaSuccess;
    runlen_sum_k<<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, scratch);
    runlen_scan_k<<<1, 1024, 0, s>>>(scratch);
    switch (esize) {
        case 1: scatter_k<uint8_t><<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, dsts, scratch); break;
        case 2: scatter_k<uint16_t><<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, dsts, scratch); break;
        case 4: scatter_k<uint32_t><<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, dsts, scratch); break;
        case 8: scatter_k<uint64_t><<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, dsts, scratch); break;
        default: return cudaErrorInvalidValue;
    }
    if (launches) *launches += 3;
    return cudaGetLastError();
}

cudaError_t chunk_merge(uint32_t* l1, const uint32_t* l2, int64_t nwords, int chunk_words_log2, const void* values,
                        int esize, const PtrList& dsts, cudaStream_t s, int64_t* launches) {
    const unsigned g = 148 * 8;
    switch (esize) {
        case 1: chunk_merge_k<uint8_t><<<g, kThreads, 0, s>>>(l1, l2, nwords, chunk_words_log2, (const uint8_t*)values, dsts); break;
        case 2: chunk_merge_k<uint16_t><<<g, kThreads, 0, s>>>(l1, l2, nwords, chunk_words_log2, (const uint16_t*)values, dsts); break;
        case 4: chunk_merge_k<uint32_t><<<g, kThreads, 0, s>>>(l1, l2, nwords, chunk_words_log2, (const uint32_t*)values, dsts); break;
        case 8: chunk_merge_k<uint64_t><<<g, kThreads, 0, s>>>(l1, l2, nwords, chunk_words_log2, (const uint64_t*)values, dsts); break;
        default: return cudaErrorInvalidValue;
    }
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t reduce_sum_i64(int64_t* acc, const PtrList& srcs, int64_t n, cudaStream_t s, int64_t* launches) {
    if (srcs.n == 0 || n == 0) return cudaSuccess;
    reduce_sum_k<<<gs_blocks(n), 256, 0, s>>>(acc, srcs, n);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t apply_add_i64(const PtrList& dsts, const int64_t* acc, int64_t n, cudaStream_t s, int64_t* launches) {
    if (dsts.n == 0 || n == 0) return cudaSuccess;
    apply_add_k<<<gs_blocks(n), 256, 0, s>>>(dsts, acc, n);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t bitmap_overlap(const uint32_t* a, const uint32_t* b, int64_t nwords, int* flag, cudaStream_t s,
                           int64_t* launches) {
    overlap_k<<<gs_blocks(nwords), 256, 0, s>>>(a, b, nwords, flag);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
