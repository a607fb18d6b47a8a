// Deep-halo body, fused (§8 row f2): h Jacobi sweeps of a tile in shared memory per launch.
//
// With halos of depth h a partition owns every input its next h sweeps depend on (the dependence
// cone of L87's window [s*i - h*C, s*(i+1) - 1 + h*C]), so the h sweeps need no exchange between
// them — and need not go through HBM either. Each CTA loads one (RB + 2h) x 128 tile of src (its
// RB x TK output rows/columns plus h halo rows and hc >= h halo columns on each side) with one
// cp.async.bulk.tensor.2d, computes levels 1..h-1 into two ping-pong shared-memory buffers
// (level t is exact on tile rows [t, RR - t) and columns [t, 128 - t); the edges beyond are never
// read by an output) and level h straight into dst. HBM traffic per h sweeps is one read and one
// write of the tile (+ the L2-resident halo overlap), so the body stops being HBM-bound: shared
// memory bandwidth and FP32 issue bound it instead (DESIGN.md f2).
//
// Arithmetic per point and level is the single-sweep kernel's, ((n + s) + (w + e)) * 0.25f with
// explicit round-to-nearest operations; points outside the update box (bounds rows [rlo, rhi),
// columns [c0, c1)) keep their value at every level. So the result is bit-identical to h
// single sweeps (tests/test_gpu_jacobi_deep.py against the oracle).
#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"
#include "track.cuh"

#include <algorithm>

namespace accmg {
namespace k {
namespace {

constexpr int W = 128;       // tile columns: one float4 per lane, one warp per row
constexpr int RB = 64;       // output rows per tile
constexpr int kMaxH = 8;
constexpr int RRmax = RB + 2 * kMaxH;
constexpr int kWarps = 8;

__device__ __forceinline__ float st5(float n, float s, float w, float e) {
    return __fmul_rn(__fadd_rn(__fadd_rn(n, s), __fadd_rn(w, e)), 0.25f);
}

__device__ __forceinline__ int64_t clamp64(int64_t v, int64_t lo, int64_t hi) { return v < lo ? lo : (v > hi ? hi : v); }

struct LevelCtx {
    unsigned upd;      // this lane's columns inside the update box (bit c: column 4*lane + c)
    unsigned onib;     // this lane's columns that are outputs of this tile
    int rlo_t, rhi_t;  // update box rows, tile-relative
    float* gdst;       // dst row of tile row 0 at this lane's first column (final level)
    int64_t cols;
    int64_t e0;        // flat index of tile row 0, tile column 0 (tracking)
};

template <bool MASK>
__device__ __forceinline__ float4 point4(const float4& N, const float4& C, const float4& S, int r, const LevelCtx& x) {
    const float w = __shfl_up_sync(dev::kFull, C.w, 1);
    const float e = __shfl_down_sync(dev::kFull, C.x, 1);
    float4 o;
    o.x = st5(N.x, S.x, w, C.y);
    o.y = st5(N.y, S.y, C.x, C.z);
    o.z = st5(N.z, S.z, C.y, C.w);
    o.w = st5(N.w, S.w, C.z, e);
    if constexpr (MASK) {
        const unsigned m = (r >= x.rlo_t && r < x.rhi_t) ? x.upd : 0u;
        o.x = (m & 1u) ? o.x : C.x;
        o.y = (m & 2u) ? o.y : C.y;
        o.z = (m & 4u) ? o.z : C.z;
        o.w = (m & 8u) ? o.w : C.w;
    }
    return o;
}

template <bool FINAL, bool MASK, bool TRACK>
__device__ __forceinline__ void emit(const float4& N, const float4& C, const float4& S, int r, float* __restrict__ out,
                                     int col, const LevelCtx& x, dev::WarpTracker<4>& trk, const Track& t) {
    const float4 o = point4<MASK>(N, C, S, r, x);
    if constexpr (!FINAL) {
        *reinterpret_cast<float4*>(out + r * W + col) = o;
    } else {
        float* p = x.gdst + (int64_t)r * x.cols;
        if (!MASK || x.onib == 0xFu) {
            if (MASK || x.onib) *reinterpret_cast<float4*>(p) = o;
        } else if (x.onib) {
            if (x.onib & 1u) p[0] = o.x;
            if (x.onib & 2u) p[1] = o.y;
            if (x.onib & 4u) p[2] = o.z;
            if (x.onib & 8u) p[3] = o.w;
        }
        if constexpr (TRACK) trk.mark(t.l1, t.l2, t.l2_shift, x.e0 + (int64_t)r * x.cols);
    }
}

// One level on tile rows [ra, rb) of this warp: in -> out (shared) or -> dst (final level). Rows
// march through three named registers unrolled by three, so no register is copied per row.
template <bool FINAL, bool MASK, bool TRACK>
__device__ __forceinline__ void level_rows(const float* __restrict__ in, float* __restrict__ out, int ra, int rb,
                                           int col, const LevelCtx& x, dev::WarpTracker<4>& trk, const Track& t) {
    if (ra >= rb) return;  // warp-uniform
    const float* q = in + col;
    float4 X0 = *reinterpret_cast<const float4*>(q + (ra - 1) * W);
    float4 X1 = *reinterpret_cast<const float4*>(q + ra * W);
    float4 X2;
    int r = ra;
    for (; r + 3 <= rb; r += 3) {
        X2 = *reinterpret_cast<const float4*>(q + (r + 1) * W);
        emit<FINAL, MASK, TRACK>(X0, X1, X2, r, out, col, x, trk, t);
        X0 = *reinterpret_cast<const float4*>(q + (r + 2) * W);
        emit<FINAL, MASK, TRACK>(X1, X2, X0, r + 1, out, col, x, trk, t);
        X1 = *reinterpret_cast<const float4*>(q + (r + 3) * W);
        emit<FINAL, MASK, TRACK>(X2, X0, X1, r + 2, out, col, x, trk, t);
    }
    if (r < rb) {
        X2 = *reinterpret_cast<const float4*>(q + (r + 1) * W);
        emit<FINAL, MASK, TRACK>(X0, X1, X2, r, out, col, x, trk, t);
        if (r + 1 < rb) {
            X0 = *reinterpret_cast<const float4*>(q + (r + 2) * W);
            emit<FINAL, MASK, TRACK>(X1, X2, X0, r + 1, out, col, x, trk, t);
        }
    }
}

template <bool MASK, bool TRACK>
__device__ __forceinline__ void levels(float* buf0, float* buf1, int h, int RR, int rfin, int warp, int col,
                                       const LevelCtx& x, dev::WarpTracker<4>& trk, const Track& t) {
    const float* in = buf0;
    float* out = buf1;
    for (int lv = 1; lv <= h; ++lv) {
        // level lv is needed on tile rows [lv, RR - lv); the final level on the output rows
        // [h, rfin) (rfin < h + RB in the last row tile)
        const int lo = lv, hi = lv == h ? rfin : RR - lv;
        const int per = (hi - lo + kWarps - 1) / kWarps;
        const int ra = lo + warp * per, rb = min(ra + per, hi);
        if (lv == h)
            level_rows<true, MASK, TRACK>(in, nullptr, ra, rb, col, x, trk, t);
        else
            level_rows<false, MASK, TRACK>(in, out, ra, rb, col, x, trk, t);
        __syncthreads();
        float* nin = out;
        out = const_cast<float*>(in);
        in = nin;
    }
}

template <bool TRACK>
__global__ void __launch_bounds__(256, 2)
jacobi2d_deep_k(const __grid_constant__ CUtensorMap map, float* __restrict__ dst, int64_t cols, int64_t r0,
                int64_t r1, int64_t rlo, int64_t rhi, int64_t c0, int64_t c1, int64_t cbase, int64_t row_lo, int h,
                int hc, Track t) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    float* buf0 = reinterpret_cast<float*>(smem_raw);
    float* buf1 = buf0 + RRmax * W;
    __shared__ __align__(8) uint64_t bar;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int TK = W - 2 * hc;
    const int RR = RB + 2 * h;
    const int64_t k0 = cbase + (int64_t)blockIdx.x * TK;  // first output column
    const int64_t kt = k0 - hc;                           // tile column 0
    const int64_t y0 = r0 + (int64_t)blockIdx.y * RB;     // first output row
    const int64_t grow0 = y0 - h;                         // tile row 0
    if (tid == 0) {
        dev::mbar_init(&bar, 1);
        dev::mbar_fence_init();
        dev::mbar_expect_tx(&bar, (uint32_t)(RR * W * 4));
        dev::tma_load_2d(&map, &bar, buf0, (int)kt, (int)(grow0 - row_lo));
    }
    __syncthreads();
    LevelCtx x;
    x.upd = 0u;
    x.onib = 0u;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        const int64_t K = kt + 4 * lane + c;
        if (K >= c0 && K < c1) {
            x.upd |= 1u << c;
            if (K >= k0 && K < k0 + TK) x.onib |= 1u << c;
        }
    }
    x.rlo_t = (int)clamp64(rlo - grow0, 0, RR);
    x.rhi_t = (int)clamp64(rhi - grow0, 0, RR);
    x.cols = cols;
    x.gdst = dst + grow0 * cols + kt + 4 * lane;
    x.e0 = grow0 * cols + kt;
    const int rfin = (int)clamp64(r1 - grow0, 0, h + RB);
    // interior tile: every point of the tile is updated, every lane's columns are outputs but
    // those of the hc/4 halo lanes on each side
    const bool interior = grow0 >= rlo && grow0 + RR <= rhi && kt >= c0 && kt + W <= c1;
    dev::WarpTracker<4> trk;
    if constexpr (TRACK) trk.init(x.onib);
    dev::mbar_wait(&bar, 0);
    const int col = 4 * lane;
    if (interior)
        levels<false, TRACK>(buf0, buf1, h, RR, rfin, warp, col, x, trk, t);
    else
        levels<true, TRACK>(buf0, buf1, h, RR, rfin, warp, col, x, trk, t);
}

}  // namespace

cudaError_t jacobi2d_deep(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                          int64_t rlo, int64_t rhi, int64_t c0, int64_t c1, int h, int64_t src_lo, int64_t src_hi,
                          Track t, cudaStream_t s, int64_t* launches) {
    if (h < 1 || h > kMaxH || cols % 4 != 0 || cols < W || cols >= (1ll << 31) ||
        (reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) % 16 != 0)
        return cudaErrorNotSupported;
    if (r1 <= r0 || c1 <= c0) return cudaSuccess;
    auto fn = tma_encode_fn();
    if (!fn) return cudaErrorNotSupported;
    const int64_t row_lo = (src_lo + cols - 1) / cols, row_hi = src_hi / cols;
    // the rows the outputs depend on (dependence cone) must lie in src's allocation
    if (row_lo > std::max<int64_t>(r0 - h, 0) || row_hi < std::min<int64_t>(r1 + h, rows)) return cudaErrorInvalidValue;
    const int hc = h <= 4 ? 4 : 8;
    const int RR = RB + 2 * h;
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)(row_hi - row_lo)};
    cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
    cuuint32_t box[2] = {(cuuint32_t)W, (cuuint32_t)RR};
    cuuint32_t es[2] = {1, 1};
    if (fn(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(src) + row_lo * cols, dims, strides, box, es,
           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return cudaErrorNotSupported;
    const int64_t cbase = (c0 / 4) * 4;
    const int TK = W - 2 * hc;
    const size_t smem = (size_t)2 * RRmax * W * 4;
    auto kern = t.l1 ? jacobi2d_deep_k<true> : jacobi2d_deep_k<false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    dim3 grid((unsigned)((c1 - cbase + TK - 1) / TK), (unsigned)((r1 - r0 + RB - 1) / RB));
    kern<<<grid, 256, smem, s>>>(map, dst, cols, r0, r1, rlo, rhi, c0, c1, cbase, row_lo, h, hc, t);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
