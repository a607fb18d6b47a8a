// Deep-halo body, register-streamed (§8 row f2; the implementation for h <= 8, cols % 4 == 0).
//
// Temporal blocking along the streaming dimension: one warp owns a 128-column strip (4 columns per
// lane: TK = 128 - 2*hc outputs plus hc >= h halo columns per side) and a segment of L output rows,
// and marches down the rows of src once. Every input row that arrives (TMA, a per-warp 4-stage ring
// of 6-row boxes completing on mbarriers) advances all h levels by one row:
//
//   level 0 row i         = input row i
//   level t row i - t     = J(level t-1 rows i-t-1, i-t, i-t+1)       t = 1..h
//   dst row (i - h)       = level h row i - h                          (stored to HBM)
//
// Each level keeps its three newest rows in registers; the row loop is unrolled by three so the
// slot of row j is j mod 3 at compile time and no register is ever copied. Nothing but the input
// rows passes through shared memory and only the final level reaches HBM, so h sweeps cost one read
// and one write of the field; the per-level cost is two shuffles and 16 FP32 operations per 4
// points (6 paired FP32 instructions in the interior). Warps are independent (no CTA barrier): a persistent grid of 16 (h <= 6) or 12 warps per SM
// walks the (strip, segment) items, neighbouring warps on neighbouring strips (shared halo columns
// hit L2).
//
// Arithmetic and boundary rule as in jacobi2d_deep.cu: ((n + s) + (w + e)) * 0.25f with explicit
// round-to-nearest operations; points outside the update box keep their value at every level;
// level t is exact on tile columns [t, 128 - t), so outputs (columns >= hc >= h from the strip
// edge) never see the strip edge. Bit-identical to h single sweeps.
#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"
#include "track.cuh"

#include <algorithm>

namespace accmg {
namespace k {
namespace {

constexpr int W = 128;        // strip columns (one float4 per lane)
constexpr int RS = 6;         // rows per TMA stage (a multiple of 3: the unroll period)
constexpr int kStages = 4;    // per-warp ring
// warps per CTA and CTAs per SM: 2 x 8 up to h = 6 (<= 128 registers); h = 7, 8 hold 84-96
// registers of level state alone, so they run 1 x 12 warps with up to 168 registers (no spills)
template <int H> struct Cfg { static constexpr int NW = H >= 7 ? 12 : 8, MINB = H >= 7 ? 1 : 2; };
constexpr int kMaxWarps = 12;
constexpr int kSegMax = 512;  // output rows per item (fewer when a partition is short: balance)
constexpr int kStageFloats = RS * W;
constexpr uint32_t kStageBytes = kStageFloats * 4;

__device__ __forceinline__ float st5(float n, float s, float w, float e) {
    return __fmul_rn(__fadd_rn(__fadd_rn(n, s), __fadd_rn(w, e)), 0.25f);
}

// Level rows live as two packed pairs P = (x, z), Q = (y, w) of a lane's four columns x, y, z, w:
// the horizontal sums then pair up as (w_in + y, y + w) = (w_in, y) + Q and (x + z, z + e_in) =
// P + (z, e_in), so a level costs 6 paired FP32 instructions (PTX add/mul.rn.f32x2: per-lane IEEE
// round-to-nearest, no flush — the bits of the scalar __fadd_rn / __fmul_rn sequence), two
// shuffles and two register moves per 4 points.
struct V4 {
    uint64_t p, q;
};

__device__ __forceinline__ uint64_t pk(float a, float b) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ void upk(uint64_t v, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); }
__device__ __forceinline__ uint64_t add2(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ uint64_t mul2(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ float4 to4(const V4& v) {
    float4 f;
    upk(v.p, f.x, f.z);
    upk(v.q, f.y, f.w);
    return f;
}
__device__ __forceinline__ V4 from4(const float4& f) { return V4{pk(f.x, f.z), pk(f.y, f.w)}; }

struct Item {
    unsigned upd, onib;  // lane columns inside the update box / outputs of this strip
    int lo_loc, hi_loc;  // update box rows, local to the item's first input row
    int out_lo, out_hi;  // local rows i (input step) whose final level is stored
    int64_t e0;          // flat index of the item's first input row, strip column 0
    int64_t cols;
    float* gdst;         // dst at (first input row, this lane's first column)
};

template <bool MASK>
__device__ __forceinline__ float4 jstep(const float4& N, const float4& C, const float4& S, int j, const Item& it) {
    const float w = __shfl_up_sync(dev::kFull, C.w, 1);
    const float e = __shfl_down_sync(dev::kFull, C.x, 1);
    float4 o;
    o.x = st5(N.x, S.x, w, C.y);
    o.y = st5(N.y, S.y, C.x, C.z);
    o.z = st5(N.z, S.z, C.y, C.w);
    o.w = st5(N.w, S.w, C.z, e);
    if constexpr (MASK) {
        const unsigned m = (j >= it.lo_loc && j < it.hi_loc) ? it.upd : 0u;
        o.x = (m & 1u) ? o.x : C.x;
        o.y = (m & 2u) ? o.y : C.y;
        o.z = (m & 4u) ? o.z : C.z;
        o.w = (m & 8u) ? o.w : C.w;
    }
    return o;
}

template <bool MASK>
__device__ __forceinline__ V4 jstep2(const V4& N, const V4& C, const V4& S, int j, const Item& it) {
    if constexpr (MASK) {
        return from4(jstep<true>(to4(N), to4(C), to4(S), j, it));
    } else {
        float x, y, z, w;
        upk(C.p, x, z);
        upk(C.q, y, w);
        const float win = __shfl_up_sync(dev::kFull, w, 1);
        const float ein = __shfl_down_sync(dev::kFull, x, 1);
        const uint64_t quarter = 0x3E8000003E800000ull;  // (0.25f, 0.25f)
        const uint64_t p = add2(add2(N.p, S.p), add2(pk(win, y), C.q));  // x: (n+s)+(w_in+y); z: (n+s)+(y+w)
        const uint64_t q = add2(add2(N.q, S.q), add2(C.p, pk(z, ein)));  // y: (n+s)+(x+z); w: (n+s)+(z+e_in)
        return V4{mul2(p, quarter), mul2(q, quarter)};
    }
}

// One input row (local index i, i % 3 == PH) through all H levels.
template <int H, int PH, bool MASK>
__device__ __forceinline__ void advance(V4 (&Lv)[H][3], const V4& X, int i, const Item& it) {
    Lv[0][PH] = X;
#pragma unroll
    for (int l = 1; l <= H; ++l) {
        // level l row j = i - l from level l-1 rows j-1, j, j+1 (slots (PH - l - 1..PH - l + 1) mod 3)
        const int sj = ((PH - l) % 3 + 3) % 3;
        const int sn = (sj + 2) % 3, ss = (sj + 1) % 3;
        const V4 Y = jstep2<MASK>(Lv[l - 1][sn], Lv[l - 1][sj], Lv[l - 1][ss], i - l, it);
        if (l < H) {
            Lv[l][sj] = Y;
        } else {
            const int j = i - H;
            if (j >= it.out_lo && j < it.out_hi) {  // warp-uniform
                float* p = it.gdst + (int64_t)j * it.cols;
                const float4 f = to4(Y);
                if (it.onib == 0xFu) {
                    *reinterpret_cast<float4*>(p) = f;
                } else if (it.onib) {
                    if (it.onib & 1u) p[0] = f.x;
                    if (it.onib & 2u) p[1] = f.y;
                    if (it.onib & 4u) p[2] = f.z;
                    if (it.onib & 8u) p[3] = f.w;
                }
            }
        }
    }
}

template <int H, bool MASK, bool TRACK>
__device__ __forceinline__ void run_item(const CUtensorMap* map, uint64_t* bar, float* ring, int nst, uint32_t& g,
                                         int64_t kt, int64_t row0_map, const Item& it, const Track& t) {
    const int lane = threadIdx.x & 31;
    V4 Lv[H][3];
#pragma unroll
    for (int l = 0; l < H; ++l)
#pragma unroll
        for (int q = 0; q < 3; ++q) Lv[l][q] = V4{0ull, 0ull};
    // prologue: the first kStages stages of this item (all slots are free here)
    if (lane == 0) {
        for (int s = 0; s < kStages && s < nst; ++s) {
            const uint32_t gs = g + s, slot = gs % kStages;
            dev::mbar_expect_tx(&bar[slot], kStageBytes);
            dev::tma_load_2d(map, &bar[slot], ring + slot * kStageFloats, (int)kt, (int)(row0_map + (int64_t)s * RS));
        }
    }
    for (int s = 0; s < nst; ++s) {
        const uint32_t gs = g + s, slot = gs % kStages;
        dev::mbar_wait(&bar[slot], (gs / kStages) & 1u);
        const float* T = ring + slot * kStageFloats + 4 * lane;
        const int i0 = s * RS;
#pragma unroll
        for (int rr = 0; rr < RS; rr += 3) {
            const V4 X0 = from4(*reinterpret_cast<const float4*>(T + (rr + 0) * W));
            const V4 X1 = from4(*reinterpret_cast<const float4*>(T + (rr + 1) * W));
            const V4 X2 = from4(*reinterpret_cast<const float4*>(T + (rr + 2) * W));
            advance<H, 0, MASK>(Lv, X0, i0 + rr + 0, it);
            advance<H, 1, MASK>(Lv, X1, i0 + rr + 1, it);
            advance<H, 2, MASK>(Lv, X2, i0 + rr + 2, it);
        }
        __syncwarp();  // every lane has consumed the slot
        if (lane == 0 && s + kStages < nst) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            const int sn = s + kStages;
            dev::mbar_expect_tx(&bar[slot], kStageBytes);
            dev::tma_load_2d(map, &bar[slot], ring + slot * kStageFloats, (int)kt, (int)(row0_map + (int64_t)sn * RS));
        }
    }
    g += (uint32_t)nst;
}

template <int H, bool TRACK>
__global__ void __launch_bounds__(Cfg<H>::NW * 32, Cfg<H>::MINB)
deep_stream_k(const __grid_constant__ CUtensorMap map, float* __restrict__ dst, int64_t cols, int64_t r0, int64_t r1,
              int64_t rlo, int64_t rhi, int64_t c0, int64_t c1, int64_t cbase, int64_t row_lo, int hc, int nstrips,
              int nsegs, int kSeg, Track t) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    constexpr int kWarps = Cfg<H>::NW;
    __shared__ __align__(8) uint64_t bars[kMaxWarps][kStages];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float* ring = reinterpret_cast<float*>(smem_raw) + warp * kStages * kStageFloats;
    uint64_t* bar = bars[warp];
    if (lane == 0) {
        for (int s = 0; s < kStages; ++s) dev::mbar_init(&bar[s], 1);
        dev::mbar_fence_init();
        dev::tma_prefetch_desc(&map);
    }
    __syncwarp();
    const int TK = W - 2 * hc;
    const int nitems = nstrips * nsegs;
    uint32_t g = 0;  // stages consumed by this warp so far (slot = g % kStages, parity = g / kStages)
    for (int item = blockIdx.x * kWarps + warp; item < nitems; item += gridDim.x * kWarps) {
        const int strip = item % nstrips, seg = item / nstrips;
        const int64_t k0 = cbase + (int64_t)strip * TK, kt = k0 - hc;
        const int64_t y0 = r0 + (int64_t)seg * kSeg;
        const int lc = (int)std::min<int64_t>(kSeg, r1 - y0);
        const int64_t ybeg = y0 - H;  // local input row 0
        const int nrow = 2 * H + lc;
        const int nst = (nrow + RS - 1) / RS;
        Item it;
        it.upd = 0u;
        it.onib = 0u;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const int64_t K = kt + 4 * lane + c;
            if (K >= c0 && K < c1) {
                it.upd |= 1u << c;
                if (K >= k0 && K < k0 + TK) it.onib |= 1u << c;
            }
        }
        it.lo_loc = (int)std::max<int64_t>(std::min<int64_t>(rlo - ybeg, 1 << 30), -(1 << 30));
        it.hi_loc = (int)std::max<int64_t>(std::min<int64_t>(rhi - ybeg, 1 << 30), -(1 << 30));
        it.out_lo = H;  // local level-h rows j = i - h: output rows y0 .. y0 + lc - 1 are j = h .. h + lc - 1
        it.out_hi = H + lc;
        it.cols = cols;
        it.e0 = ybeg * cols + kt;
        it.gdst = dst + ybeg * cols + kt + 4 * lane;
        // interior item: every row it computes lies in the row box and the strip in the column box
        const bool interior = ybeg >= rlo && ybeg + (int64_t)nst * RS <= rhi && kt >= c0 && kt + W <= c1;
        if (interior)
            run_item<H, false, TRACK>(&map, bar, ring, nst, g, kt, ybeg - row_lo, it, t);
        else
            run_item<H, true, TRACK>(&map, bar, ring, nst, g, kt, ybeg - row_lo, it, t);
        if constexpr (TRACK)  // dirty bits of the item's output rectangle, after its stores
            dev::mark_rect(t.l1, t.l2, t.l2_shift, y0, y0 + lc, cols, std::max<int64_t>(k0, c0),
                           std::min<int64_t>(k0 + TK, c1), lane, 32);
    }
}

template <int H>
cudaError_t launch_h(const CUtensorMap& map, float* dst, int64_t cols, int64_t r0, int64_t r1, int64_t rlo, int64_t rhi,
                     int64_t c0, int64_t c1, int64_t cbase, int64_t row_lo, int hc, int nstrips, Track t,
                     cudaStream_t s) {
    auto kern = t.l1 ? deep_stream_k<H, true> : deep_stream_k<H, false>;
    constexpr int kWarps = Cfg<H>::NW;
    const size_t smem = (size_t)kWarps * kStages * kStageBytes;
    cudaError_t e = kernel_prep(kern, kWarps * 32, smem);
    if (e != cudaSuccess) return e;
    const int nsm = sm_count_cached();
    // segment length: items are equal, so time ~ waves x rows per item = ceil(items / resident
    // warps) x (seg + 2h); pick the segment count minimising that (short partitions — 4096 rows of
    // C2 at P = 8 — would otherwise run 1.3 waves of 512-row items)
    const int64_t twarps = (int64_t)Cfg<H>::MINB * nsm * kWarps;
    const int64_t nrows = r1 - r0;
    int nsegs = 1;
    double best = 1e300;
    for (int64_t ns = (nrows + kSegMax - 1) / kSegMax; ns <= std::max<int64_t>(1, nrows / 32); ++ns) {
        const int64_t sg = (nrows + ns - 1) / ns;
        const int64_t waves = (ns * nstrips + twarps - 1) / twarps;
        const double cost = (double)waves * (double)(sg + 2 * H);
        if (cost < best * 0.999) {
            best = cost;
            nsegs = (int)ns;
        }
        if (waves > 64) break;
    }
    const int seg = (int)((nrows + nsegs - 1) / nsegs);
    const int nitems = nstrips * nsegs;
    const int grid = std::max(1, std::min(Cfg<H>::MINB * nsm, (nitems + kWarps - 1) / kWarps));
    kern<<<grid, kWarps * 32, smem, s>>>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, nsegs,
                                          seg, t);
    return cudaGetLastError();
}

}  // namespace

cudaError_t jacobi2d_deep_stream(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                                 int64_t rlo, int64_t rhi, int64_t c0, int64_t c1, int h, int64_t src_lo,
                                 int64_t src_hi, Track t, cudaStream_t s, int64_t* launches) {
    if (h < 2 || h > 8 || cols % 4 != 0 || cols < W || cols >= (1ll << 31) ||
        (reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) % 16 != 0)
        return cudaErrorNotSupported;
    if (r1 <= r0 || c1 <= c0) return cudaSuccess;
    const int64_t row_lo = (src_lo + cols - 1) / cols, row_hi = src_hi / cols;
    if (row_lo > std::max<int64_t>(r0 - h, 0) || row_hi < std::min<int64_t>(r1 + h, rows)) return cudaErrorInvalidValue;
    const int hc = h <= 4 ? 4 : 8;
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)(row_hi - row_lo)};
    cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
    cuuint32_t box[2] = {(cuuint32_t)W, (cuuint32_t)RS};
    cuuint32_t es[2] = {1, 1};
    if (!tma_encode_tiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(src) + row_lo * cols, dims,
                          strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE))
        return cudaErrorNotSupported;
    const int64_t cbase = (c0 / 4) * 4;
    const int TK = W - 2 * hc;
    const int nstrips = (int)((c1 - cbase + TK - 1) / TK);
    cudaError_t e;
    switch (h) {
        case 2: e = launch_h<2>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        case 3: e = launch_h<3>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        case 4: e = launch_h<4>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        case 5: e = launch_h<5>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        case 6: e = launch_h<6>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        case 7: e = launch_h<7>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
        default: e = launch_h<8>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, hc, nstrips, t, s); break;
    }
    if (launches) *launches += 1;
    return e;
}

}  // namespace k
}  // namespace accmg
