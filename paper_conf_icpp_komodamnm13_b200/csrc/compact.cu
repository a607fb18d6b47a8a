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
// scan (one block: tile offsets + header; clears L2), write (warp ballots + popc prefix sums;
// coalesced gathers of the payload; clears L1 as it goes). HBM-bound: per dirty element
// 1/8 B bitmap + esize read + esize written, + 16 B per run.
#include "kernels.h"
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
    if (ws < w1) {
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
// (coalesced loads, warp-shuffle scans, one carry per step), then the L2 popcount + clear.
__global__ void __launch_bounds__(1024)
scan_k(const int64_t* __restrict__ tile_counts, int64_t ntiles, int64_t* __restrict__ tile_offs,
       int64_t* __restrict__ totals, uint32_t* __restrict__ l2, int64_t nl2words) {
    __shared__ int64_t wsum[3][32];
    __shared__ int64_t carry[3];
    __shared__ unsigned long long nchunks;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid < 3) carry[tid] = 0;
    if (tid == 0) nchunks = 0ull;
    __syncthreads();
    for (int64_t base = 0; base < ntiles; base += 1024) {
        const int64_t t = base + tid;
        int64_t v[3], inc[3];
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            v[q] = t < ntiles ? tile_counts[3 * t + q] : 0;
            inc[q] = warp_incl_scan(v[q]);
            if (lane == 31) wsum[q][warp] = inc[q];
        }
        __syncthreads();
        if (warp == 0) {
#pragma unroll
            for (int q = 0; q < 3; ++q) {
                const int64_t x = wsum[q][lane];
                const int64_t xi = warp_incl_scan(x);
                wsum[q][lane] = xi - x;  // exclusive warp offsets
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 3; ++q)
            if (t < ntiles) tile_offs[3 * t + q] = carry[q] + wsum[q][warp] + inc[q] - v[q];
        __syncthreads();
        if (tid == 1023) {
#pragma unroll
            for (int q = 0; q < 3; ++q) carry[q] += wsum[q][31] + inc[q];
        }
        __syncthreads();
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

template <typename T>
__global__ void __launch_bounds__(kThreads)
write_k(uint32_t* __restrict__ l1, int64_t nwords, const int64_t* __restrict__ tile_counts,
        const int64_t* __restrict__ tile_offs, const uint32_t* __restrict__ tile_edges, int64_t ntiles,
        const T* __restrict__ values, uint8_t* __restrict__ packed, int64_t n_runs) {
    const int64_t t = blockIdx.x;
    if (tile_counts[3 * t + 2] == 0) return;  // clean tile (no dirty element)
    const int64_t w0 = t * kTileWords;
    const int64_t nw = (w0 + kTileWords < nwords ? w0 + kTileWords : nwords) - w0;
    __shared__ uint32_t sw[kTileWords + 2];
    __shared__ int64_t woff[3][kThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int64_t i = tid; i < nw; i += kThreads) {
        sw[i + 1] = l1[w0 + i];
        l1[w0 + i] = 0u;  // clear as we go (this tile's words are read by this block only)
    }
    if (tid == 0) {
        sw[0] = t > 0 ? tile_edges[2 * (t - 1) + 1] : 0u;
        sw[nw + 1] = t + 1 < ntiles ? tile_edges[2 * (t + 1)] : 0u;
    }
    __syncthreads();
    // per-warp counts over its 256 words (lane-contiguous groups of 8)
    const int64_t wb = (int64_t)warp * (kTileWords / (kThreads / 32));  // 256 words per warp
    int64_t cs = 0, ce = 0, cel = 0;
    for (int j = 0; j < 8; ++j) {
        const int64_t i = wb + lane * 8 + j;
        if (i < nw) {
            const uint32_t w = sw[i + 1];
            cs += __popc(start_mask(w, sw[i]));
            ce += __popc(end_mask(w, sw[i + 2]));
            cel += __popc(w);
        }
    }
    cs = warp_sum(cs); ce = warp_sum(ce); cel = warp_sum(cel);
    if (lane == 0) { woff[0][warp] = cs; woff[1][warp] = ce; woff[2][warp] = cel; }
    __syncthreads();
    int64_t os = tile_offs[3 * t], oe = tile_offs[3 * t + 1], oel = tile_offs[3 * t + 2];
    for (int i = 0; i < warp; ++i) { os += woff[0][i]; oe += woff[1][i]; oel += woff[2][i]; }
    int64_t* run_start = reinterpret_cast<int64_t*>(packed + 16);
    int64_t* run_end = run_start + n_runs;
    T* payload = reinterpret_cast<T*>(packed + 16 + 16 * n_runs);
    // 8 groups of 32 words, one word per lane, in element order
    for (int g = 0; g < 8; ++g) {
        const int64_t i = wb + g * 32 + lane;
        const bool ok = i < nw;
        const uint32_t w = ok ? sw[i + 1] : 0u;
        if (__ballot_sync(dev::kFull, w != 0u) == 0u) continue;
        const uint32_t sm = ok ? start_mask(w, sw[i]) : 0u;
        const uint32_t em = ok ? end_mask(w, sw[i + 2]) : 0u;
        const int64_t gw = w0 + i;
        const int ps = __popc(sm), pe = __popc(em), pel = __popc(w);
        const int is = warp_incl_scan(ps), ie = warp_incl_scan(pe), iel = warp_incl_scan(pel);
        int64_t ks = os + is - ps, ke = oe + ie - pe;
        for (uint32_t m = sm; m; m &= m - 1) run_start[ks++] = gw * 32 + (__ffs(m) - 1);
        for (uint32_t m = em; m; m &= m - 1) run_end[ke++] = gw * 32 + __ffs(m);
        const int rel_el = iel - pel;  // this lane's word: first payload slot relative to oel
        // payload: word by word, lanes = element bits; all 32 words of the group are loaded before
        // any is stored (32 coalesced 128-byte loads in flight per warp: the gather is
        // latency-bound otherwise)
        const int64_t gbase = w0 + wb + g * 32;
#pragma unroll 1
        for (int q0 = 0; q0 < 32; q0 += 32) {
            uint32_t wq[32];
            int bq[32];
            T v[32];
#pragma unroll
            for (int u = 0; u < 32; ++u) {
                wq[u] = __shfl_sync(dev::kFull, w, q0 + u);
                bq[u] = __shfl_sync(dev::kFull, rel_el, q0 + u);
                v[u] = ((wq[u] >> lane) & 1u) ? values[(gbase + q0 + u) * 32 + lane] : T(0);
            }
#pragma unroll
            for (int u = 0; u < 32; ++u)
                if ((wq[u] >> lane) & 1u) payload[oel + bq[u] + __popc(wq[u] & ((1u << lane) - 1u))] = v[u];
        }
        os += __shfl_sync(dev::kFull, is, 31);
        oe += __shfl_sync(dev::kFull, ie, 31);
        oel += __shfl_sync(dev::kFull, iel, 31);
    }
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

__global__ void __launch_bounds__(32) runlen_scan_k(int64_t* __restrict__ scratch) {
    if (threadIdx.x == 0) {
        int64_t run = 0;
        for (int b = 0; b < kScatterBlocks; ++b) { scratch[kScatterBlocks + b] = run; run += scratch[b]; }
    }
}

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
    __shared__ int64_t carry;
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
        __syncthreads();
        if (tid == kThreads - 1) carry += wo + inc;
        const int nr = (int)((hi - base) < kThreads ? (hi - base) : kThreads);
        for (int q = warp; q < nr; q += kThreads / 32) {
            const int64_t st = s_start[q], ln = s_len[q], of = s_off[q];
            // 8 independent loads per lane in flight, then the stores to every destination
            for (int64_t x0 = 0; x0 < ln; x0 += 32 * 8) {
                T v[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) {
                    const int64_t x = x0 + 32 * u + lane;
                    v[u] = x < ln ? payload[of + x] : T(0);
                }
                for (int d = 0; d < dsts.n; ++d) {
                    T* dp = static_cast<T*>(dsts.p[d]) + st;
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int64_t x = x0 + 32 * u + lane;
                        if (x < ln) dp[x] = v[u];
                    }
                }
            }
        }
        __syncthreads();
    }
}

// The paper's protocol (L133-135): for every chunk whose second-level bit is set, the whole chunk's
// first-level bits decide which elements overwrite the peers' copies ("merged by the dirty bits").
// One block per dirty chunk; lanes = bits of one word; clears the chunk's L1 words afterwards.
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
        for (int64_t w = w0 + warp; w < w1; w += kThreads / 32) {
            const uint32_t m = l1[w];
            if ((m >> lane) & 1u) {
                const T v = src[w * 32 + lane];
                for (int d = 0; d < dsts.n; ++d) static_cast<T*>(dsts.p[d])[w * 32 + lane] = v;
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

cudaError_t compact_write(uint32_t* l1, int64_t nwords, int64_t ntiles, const int64_t* tile_counts,
                          const int64_t* tile_offs, const uint32_t* tile_edges, const void* values,
                          int esize, uint8_t* packed, int64_t n_runs, cudaStream_t s, int64_t* launches) {
    dim3 g((unsigned)ntiles);
    switch (esize) {
        case 1: write_k<uint8_t><<<g, kThreads, 0, s>>>(l1, nwords, tile_counts, tile_offs, tile_edges, ntiles, (const uint8_t*)values, packed, n_runs); break;
        case 2: write_k<uint16_t><<<g, kThreads, 0, s>>>(l1, nwords, tile_counts, tile_offs, tile_edges, ntiles, (const uint16_t*)values, packed, n_runs); break;
        case 4: write_k<uint32_t><<<g, kThreads, 0, s>>>(l1, nwords, tile_counts, tile_offs, tile_edges, ntiles, (const uint32_t*)values, packed, n_runs); break;
        case 8: write_k<uint64_t><<<g, kThreads, 0, s>>>(l1, nwords, tile_counts, tile_offs, tile_edges, ntiles, (const uint64_t*)values, packed, n_runs); break;
        default: return cudaErrorInvalidValue;
    }
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t scatter_packed(const uint8_t* packed, int64_t n_runs, const PtrList& dsts, int esize,
                           int64_t* scratch, cudaStream_t s, int64_t* launches) {
    if (n_runs == 0 || dsts.n == 0) return cudaSuccess;
    runlen_sum_k<<<kScatterBlocks, kThreads, 0, s>>>(packed, n_runs, scratch);
    runlen_scan_k<<<1, 32, 0, s>>>(scratch);
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
    const unsigned g = 148 * 4;
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
