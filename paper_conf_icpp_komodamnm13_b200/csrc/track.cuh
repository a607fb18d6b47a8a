// Fused write-tracking epilogue (north star (3); paper L110, L133-135 §IV.D.1): "the translator
// inserts the additional operations to turn on the dirty bits for every writes accesses to the
// replicated arrays", with a second-level bit per constant-size chunk.
//
// Warp-aggregated: a warp that wrote a contiguous span of 32*VEC elements (lane l owns elements
// E0 + VEC*l + k, k < VEC, written iff bit k of its mask) builds the span's bit pattern with
// VEC ballots, shifts it onto the absolute uint32 words and issues at most VEC+1 atomicOr
// (one per touched word) instead of one per element. Every written element sets its bit
// (also when the value is unchanged, reading G12); no bit is ever dropped because concurrent
// writers of a word combine through atomicOr.
#pragma once
#include <cstdint>

namespace accmg {
namespace dev {

constexpr unsigned kFull = 0xffffffffu;

// bit m of an 8-bit value -> bit 4m
__device__ __forceinline__ uint32_t spread4(uint32_t x) {
    x &= 0xffu;
    x = (x | (x << 12)) & 0x000F000Fu;
    x = (x | (x << 6)) & 0x03030303u;
    x = (x | (x << 3)) & 0x11111111u;
    return x;
}

// Sets chunk bit c. Thousands of warps write into one chunk and all of them would hit the same
// L2 word with an atomic, serialising at that L2 slice (measured: it doubled the tracked sweep);
// reading the word first (L2-cached load) skips the atomic once some warp has set the bit.
// A stale 0 only costs one redundant atomicOr; bits are cleared only by the compaction kernels,
// which are stream-ordered after this kernel.
__device__ __forceinline__ void set_chunk_bit(uint32_t* l2, int64_t c) {
    const uint32_t bit = 1u << (c & 31);
    if (!(__ldcg(l2 + (c >> 5)) & bit)) atomicOr(l2 + (c >> 5), bit);
}

// Sets the L2 (chunk) bits of elements [first, last] (inclusive, all written). `cache` holds the
// last chunk this warp marked so steady marching re-issues nothing.
__device__ __forceinline__ void track_l2(uint32_t* l2, int l2_shift, int64_t first, int64_t last, int64_t& cache) {
    int64_t c0 = first >> l2_shift, c1 = last >> l2_shift;
    if (c0 == c1 && c0 == cache) return;
    for (int64_t c = c0; c <= c1; ++c) set_chunk_bit(l2, c);
    cache = c1;
}

// VEC = 4: lane l owns elements E0 + 4l + k (k < 4), written iff (nib >> k) & 1.
// VEC = 1: lane l owns element E0 + l, written iff nib & 1.
// Must be called by all 32 lanes of the warp (warp-uniform E0).
template <int VEC>
__device__ __forceinline__ void track_warp(uint32_t* __restrict__ l1, uint32_t* __restrict__ l2, int l2_shift,
                                           int64_t E0, unsigned nib, int64_t& l2_cache) {
    const int lane = threadIdx.x & 31;
    uint32_t rel[VEC];
    if (VEC == 4) {
        uint32_t b0 = __ballot_sync(kFull, nib & 1u), b1 = __ballot_sync(kFull, nib & 2u);
        uint32_t b2 = __ballot_sync(kFull, nib & 4u), b3 = __ballot_sync(kFull, nib & 8u);
        if ((b0 | b1 | b2 | b3) == 0u) return;
#pragma unroll
        for (int q = 0; q < VEC; ++q) {
            int sh = 8 * q;
            rel[q] = spread4(b0 >> sh) | (spread4(b1 >> sh) << 1) | (spread4(b2 >> sh) << 2) |
                     (spread4(b3 >> sh) << 3);
        }
    } else {
        rel[0] = __ballot_sync(kFull, nib & 1u);
        if (rel[0] == 0u) return;
    }
    const int s = (int)(E0 & 31);
    const int64_t w0 = E0 >> 5;
    // absolute word q (0..VEC) of the span
    if (lane <= VEC) {
        uint32_t lo = 0u, hi = 0u;  // rel[lane], rel[lane-1] without dynamic register indexing
#pragma unroll
        for (int q = 0; q < VEC; ++q) {
            lo = (q == lane) ? rel[q] : lo;
            hi = (q == lane - 1) ? rel[q] : hi;
        }
        uint32_t v = (lo << s) | (s ? (hi >> (32 - s)) : 0u);
        if (v) atomicOr(l1 + w0 + lane, v);
    }
    if (lane == 0) {
        // first and last written element of the span
        int f = -1, l = -1;
#pragma unroll
        for (int q = 0; q < VEC; ++q) {
            if (rel[q]) {
                if (f < 0) f = 32 * q + __ffs(rel[q]) - 1;
                l = 32 * q + 31 - __clz(rel[q]);
            }
        }
        track_l2(l2, l2_shift, E0 + f, E0 + l, l2_cache);
    }
}

// Row-marching variant: a warp that writes the same lane/element mask on many rows (a fixed
// column strip) builds the span pattern once; each row then costs one shift, plain stores for
// the words it owns outright and atomicOr only on shared edge words, plus a cached L2 check.
// Precondition: the elements a warp writes in one row form one contiguous range that no other
// warp writes in the same loop (true for the row-strip bodies).
template <int VEC>
struct WarpTracker {
    uint32_t lo = 0u, hi = 0u;  // this lane's relative words rel[lane], rel[lane-1]
    int first = -1, last = -1;  // first/last written element offset within the span
    int64_t l2_cache = -1;

    __device__ __forceinline__ void init(unsigned nib) {
        const int lane = threadIdx.x & 31;
        uint32_t rel[VEC];
        if constexpr (VEC == 4) {
            uint32_t b0 = __ballot_sync(kFull, nib & 1u), b1 = __ballot_sync(kFull, nib & 2u);
            uint32_t b2 = __ballot_sync(kFull, nib & 4u), b3 = __ballot_sync(kFull, nib & 8u);
#pragma unroll
            for (int q = 0; q < VEC; ++q) {
                const int sh = 8 * q;
                rel[q] = spread4(b0 >> sh) | (spread4(b1 >> sh) << 1) | (spread4(b2 >> sh) << 2) |
                         (spread4(b3 >> sh) << 3);
            }
        } else {
            rel[0] = __ballot_sync(kFull, nib & 1u);
        }
#pragma unroll
        for (int q = 0; q < VEC; ++q) {
            lo = (q == lane) ? rel[q] : lo;
            hi = (q == lane - 1) ? rel[q] : hi;
            if (rel[q]) {
                if (first < 0) first = 32 * q + __ffs(rel[q]) - 1;
                last = 32 * q + 31 - __clz(rel[q]);
            }
        }
    }

    // All rows [rs, re) of a strip at once, after the stencil loop (keeps the tracking work out of
    // the load pipeline): lane i handles (row, word) pair i, 32 at a time; each row's chunk range is
    // marked once unless the previous row already marked it.
    __device__ __forceinline__ void mark_rows(uint32_t* __restrict__ l1, uint32_t* __restrict__ l2, int l2_shift,
                                              int64_t rs, int64_t re, int64_t cols, int64_t cw) {
        if (first < 0) return;
        const int lane = threadIdx.x & 31;
        constexpr int NW = VEC + 1;
        const int64_t n = (re - rs) * NW;
        for (int64_t base = 0; base < n; base += 32) {  // warp-uniform trip count (shuffles)
            const int64_t i = base + lane;
            const bool ok = i < n;
            const int64_t r = rs + i / NW;
            const int q = (int)(i % NW);
            // lane k (< VEC) holds rel[k] in `lo`; lane VEC holds 0
            const uint32_t lo_q = __shfl_sync(kFull, lo, q);
            const uint32_t hi_q = __shfl_sync(kFull, lo, q == 0 ? 31 : q - 1);  // lane 31 holds 0
            if (!ok) continue;
            const int64_t E0 = r * cols + cw;
            const int s = (int)(E0 & 31);
            const uint32_t v = (lo_q << s) | (s ? (hi_q >> (32 - s)) : 0u);
            const int64_t w = (E0 >> 5) + q;
            const bool inner = w * 32 >= E0 + first && w * 32 + 31 <= E0 + last;
            if (v) {
                if (inner) l1[w] = v;
                else atomicOr(l1 + w, v);
            }
            if (q == 0) {
                const int64_t c0 = (E0 + first) >> l2_shift, c1 = (E0 + last) >> l2_shift;
                const int64_t cp = r > rs ? (E0 - cols + last) >> l2_shift : -1;
                for (int64_t c = c0; c <= c1; ++c)
                    if (c != cp) set_chunk_bit(l2, c);
            }
        }
    }

    __device__ __forceinline__ void mark(uint32_t* __restrict__ l1, uint32_t* __restrict__ l2, int l2_shift,
                                         int64_t E0) {
        if (first < 0) return;  // warp-uniform: nothing written by this warp
        const int lane = threadIdx.x & 31;
        const int s = (int)(E0 & 31);
        if (lane <= VEC) {
            const uint32_t v = (lo << s) | (s ? (hi >> (32 - s)) : 0u);
            const int64_t w = (E0 >> 5) + lane;
            // A word lying entirely inside this warp's written range holds only elements this warp
            // writes (the range is contiguous and no other warp writes them in this loop, L62), and
            // compaction left it zero: a plain store is exact. Edge words may be shared: atomicOr.
            const bool inner = w * 32 >= E0 + first && w * 32 + 31 <= E0 + last;
            if (v) {
                if (inner) l1[w] = v;
                else atomicOr(l1 + w, v);
            }
        }
        if (lane == 0) track_l2(l2, l2_shift, E0 + first, E0 + last, l2_cache);
    }
};

// Block-level epilogue for a CTA that wrote every element of the rectangle rows [rs, re) x
// columns [ca, cb) of a row-major array with `cols` columns (and nothing else in this loop); with
// nplanes > 1 the same rectangle repeated every `pstride` rows (a 3-D block: planes of a
// [n0*n1][n2] view). All threads of the block (tid < nthr) call it once after their stores.
// Thread i handles (row, word) pair i, so one warp-wide store covers 32 words of several rows
// instead of one mark per row and warp. A word lying entirely inside one row's written range holds
// only this CTA's elements and was cleared by the last compaction: plain store. Words shared with a
// neighbouring CTA: atomicOr. Each row's chunk bits are set unless the previous row of the same
// plane already set them (check-first atomics).
__device__ __forceinline__ void mark_rect(uint32_t* __restrict__ l1, uint32_t* __restrict__ l2, int l2_shift, int64_t rs,
                                          int64_t re, int64_t cols, int64_t ca, int64_t cb, int tid, int nthr,
                                          int nplanes = 1, int64_t pstride = 0) {
    if (rs >= re || ca >= cb || nplanes < 1) return;
    const int nr = (int)(re - rs);
    const int nwr = (int)((cb - ca + 31) >> 5) + 1;  // words one row can touch
    const int npairs = nplanes * nr * nwr;
    for (int i = tid; i < npairs; i += nthr) {
        const int row = i / nwr, q = i - row * nwr;
        const int pl = row / nr, dr = row - pl * nr;
        const int64_t e0 = (rs + pl * pstride + dr) * cols + ca, e1 = e0 + (cb - ca);
        const int64_t w = (e0 >> 5) + q;
        if (w * 32 >= e1) continue;
        const int64_t lo = e0 > w * 32 ? e0 : w * 32, hi = e1 < w * 32 + 32 ? e1 : w * 32 + 32;
        const int blo = (int)(lo - w * 32), n = (int)(hi - lo);
        const uint32_t v = (n == 32 ? 0xffffffffu : ((1u << n) - 1u)) << blo;
        if (n == 32) l1[w] = v;
        else atomicOr(l1 + w, v);
    }
    for (int row = tid; row < nplanes * nr; row += nthr) {
        const int pl = row / nr, dr = row - pl * nr;
        const int64_t e0 = (rs + pl * pstride + dr) * cols + ca;
        int64_t c0 = e0 >> l2_shift;
        const int64_t c1 = (e0 + (cb - ca) - 1) >> l2_shift;
        if (dr > 0 && c0 == ((e0 - cols + (cb - ca) - 1) >> l2_shift)) ++c0;  // previous row set it
        for (int64_t c = c0; c <= c1; ++c) set_chunk_bit(l2, c);
    }
}

}  // namespace dev
}  // namespace accmg
