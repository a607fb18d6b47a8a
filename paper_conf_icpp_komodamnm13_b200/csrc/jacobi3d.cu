// Loop body: 3-D 7-point Jacobi sweep (§8 row f2: the multi-dimensional stencils of L256, with
// plane-block partitioning — declared windows stride = n1*n2, left = right = n1*n2).
//
//   dst[i][j][k] = ((((u + d) + (n + s)) + ((w + e) + (c + c))) * 0.125f
//   u/d = src[i-1/i+1][j][k], n/s = src[i][j-1/j+1][k], w/e = src[i][j][k-1/k+1], c = src[i][j][k]
//   (damped Jacobi of the 3-D Laplacian; reading in DESIGN.md), interior points only.
//
// TMA-staged shared-memory tiles (B200): each CTA owns a 16 (j) x 128 (k) column of the domain and
// marches down a segment of planes i. One thread issues cp.async.bulk.tensor.3d loads of
// 18 x 136-float tiles (the tile plus its j and k halo) of successive planes into a 4-stage ring
// completed on mbarriers, so three planes are resident while the fourth streams in; every input
// element crosses HBM once (+ the 2 halo rows / 2 halo planes per segment, L2-resident). Threads
// read the 7 operands from shared memory (horizontal neighbours by warp shuffle), use explicit
// round-to-nearest adds in the stated order, and store 128-bit vectors of interior points. The
// optional fused epilogue sets the two-level dirty bits (L133-135) once per CTA after its stores
// (mark_rect over its planes: owned words by plain stores, words shared with neighbours by atomicOr).
#include <cstdlib>

#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"
#include "track.cuh"

namespace accmg {
namespace k {
namespace {

constexpr int TK = 128;          // k columns per CTA (32 lanes x float4)
constexpr int BOXK = TK + 8;     // k halo: 4 on each side (keeps 16-byte alignment)
// TJ: j rows per CTA (8 warps x TJ/8 rows); SEG: planes per CTA. Tile = (TJ + 2) x BOXK floats.
template <int TJ, int kStages>
struct Geo {
    static constexpr int BOXJ = TJ + 2;  // j halo: 1 on each side
    static constexpr uint32_t kTileBytes = BOXK * BOXJ * 4;
    static constexpr int kStageFloats = ((kTileBytes + 127) / 128) * 32;  // TMA destinations 128-B aligned
    static constexpr size_t kSmem = (size_t)kStages * kStageFloats * 4 + kStages * 8 + 128;
};

__device__ __forceinline__ float s7(float u, float d, float n, float s, float w, float e, float c) {
    const float ud = __fadd_rn(u, d), ns = __fadd_rn(n, s), we = __fadd_rn(w, e), cc = __fadd_rn(c, c);
    return __fmul_rn(__fadd_rn(__fadd_rn(ud, ns), __fadd_rn(we, cc)), 0.125f);
}

template <bool TRACK, int TJ, int kPlaneSeg, int kStages>
__global__ void __launch_bounds__(256)
jacobi3d_tma(const __grid_constant__ CUtensorMap map, float* __restrict__ dst, int64_t n1, int64_t n2, int64_t i0,
             int64_t i1, int64_t jl, int64_t jh, int64_t kl, int64_t kh, int64_t kbase, int64_t plane_lo, Track t) {
    using G = Geo<TJ, kStages>;
    constexpr int BOXJ = G::BOXJ;
    constexpr uint32_t kTileBytes = G::kTileBytes;
    extern __shared__ __align__(128) unsigned char smem3[];
    float(*tile)[G::kStageFloats] = reinterpret_cast<float(*)[G::kStageFloats]>(
        smem3 + ((128 - (dev::smem_u32(smem3) & 127)) & 127));
    uint64_t* bar = reinterpret_cast<uint64_t*>(&tile[kStages][0]);
    (void)BOXJ;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t k0 = kbase + (int64_t)blockIdx.x * TK;
    const int64_t j0 = jl + (int64_t)blockIdx.y * TJ;
    const int64_t ps = i0 + (int64_t)blockIdx.z * kPlaneSeg;
    const int64_t pe = ps + kPlaneSeg < i1 ? ps + kPlaneSeg : i1;
    const int count = (int)(pe - ps + 2);  // planes ps-1 .. pe
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) dev::mbar_init(&bar[s], 1);
        dev::mbar_fence_init();
        dev::tma_prefetch_desc(&map);
        for (int q = 0; q < kStages && q < count; ++q) {  // all stages free at the start
            dev::mbar_expect_tx(&bar[q], kTileBytes);
            dev::tma_load_3d(&map, &bar[q], tile[q], (int)(k0 - 4), (int)(j0 - 1), (int)(ps - 1 + q - plane_lo));
        }
    }
    __syncthreads();
    // this thread's columns and rows
    const int64_t k = k0 + 4 * lane;
    unsigned nib = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c) nib |= (k + c >= kl && k + c < kh) ? (1u << c) : 0u;
    const bool full = nib == 0xFu;
    const int col = 4 + 4 * lane;  // tile column of k
    dev::mbar_wait(&bar[0], 0);
    dev::mbar_wait(&bar[1], 0);
    for (int64_t i = ps; i < pe; ++i) {
        const int q = (int)(i - ps) + 2;  // plane i+1
        dev::mbar_wait_sleep(&bar[q % kStages], (uint32_t)((q / kStages) & 1));
        const float* P0 = tile[(q - 2) % kStages];
        const float* P1 = tile[(q - 1) % kStages];
        const float* P2 = tile[q % kStages];
#pragma unroll
        for (int r = 0; r < TJ / 8; ++r) {
            const int tr = (TJ / 8) * warp + r + 1;  // tile row of j
            const int64_t j = j0 + tr - 1;
            const float4 C = *reinterpret_cast<const float4*>(P1 + tr * BOXK + col);
            const float4 N = *reinterpret_cast<const float4*>(P1 + (tr - 1) * BOXK + col);
            const float4 S = *reinterpret_cast<const float4*>(P1 + (tr + 1) * BOXK + col);
            const float4 U = *reinterpret_cast<const float4*>(P0 + tr * BOXK + col);
            const float4 D = *reinterpret_cast<const float4*>(P2 + tr * BOXK + col);
            float w = __shfl_up_sync(dev::kFull, C.w, 1);
            float e = __shfl_down_sync(dev::kFull, C.x, 1);
            if (lane == 0) w = P1[tr * BOXK + col - 1];
            if (lane == 31) e = P1[tr * BOXK + col + 4];
            const bool rowok = j < jh;  // warp-uniform
            if (rowok) {
                float o[4];
                o[0] = s7(U.x, D.x, N.x, S.x, w, C.y, C.x);
                o[1] = s7(U.y, D.y, N.y, S.y, C.x, C.z, C.y);
                o[2] = s7(U.z, D.z, N.z, S.z, C.y, C.w, C.z);
                o[3] = s7(U.w, D.w, N.w, S.w, C.z, e, C.w);
                float* out = dst + (i * n1 + j) * n2 + k;
                if (full) {
                    *reinterpret_cast<float4*>(out) = make_float4(o[0], o[1], o[2], o[3]);
                } else {
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (nib & (1u << c)) out[c] = o[c];
                }
            }
        }
        __syncthreads();  // every thread is done with plane i-1 (stage (q-2) % kStages)
        if (tid == 0 && q + kStages - 2 < count) {  // the stage of plane i-1 takes plane i-1+kStages
            const int qn = q + kStages - 2;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            dev::mbar_expect_tx(&bar[qn % kStages], kTileBytes);
            dev::tma_load_3d(&map, &bar[qn % kStages], tile[qn % kStages], (int)(k0 - 4), (int)(j0 - 1),
                             (int)(ps - 1 + qn - plane_lo));
        }
    }
    if constexpr (TRACK) {  // dirty bits of the CTA's 16 x 128 column in each of its planes, after its stores
        const int64_t je = j0 + TJ < jh ? j0 + TJ : jh, ka = k0 > kl ? k0 : kl, kb = k0 + TK < kh ? k0 + TK : kh;
        dev::mark_rect(t.l1, t.l2, t.l2_shift, ps * n1 + j0, ps * n1 + je, n2, ka, kb, tid, 256, (int)(pe - ps), n1);
    }
}

template <int TJ, int SEG, int NS = 4>
cudaError_t launch3d(const CUtensorMap& map, float* dst, int64_t n1, int64_t n2, int64_t i0, int64_t i1, int64_t jl,
                     int64_t jh, int64_t kl, int64_t kh, int64_t plane_lo, Track t, cudaStream_t s, int64_t* launches) {
    const int64_t kbase = (kl / 4) * 4;
    dim3 grid((unsigned)((kh - kbase + TK - 1) / TK), (unsigned)((jh - jl + TJ - 1) / TJ),
              (unsigned)((i1 - i0 + SEG - 1) / SEG));
    const size_t smem = Geo<TJ, NS>::kSmem;
    auto kern = t.l1 ? jacobi3d_tma<true, TJ, SEG, NS> : jacobi3d_tma<false, TJ, SEG, NS>;
    cudaError_t e = kernel_prep(kern, 256, smem);
    if (e != cudaSuccess) return e;
    kern<<<grid, 256, smem, s>>>(map, dst, n1, n2, i0, i1, jl, jh, kl, kh, kbase, plane_lo, t);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace

cudaError_t jacobi3d(const float* src, float* dst, int64_t n0, int64_t n1, int64_t n2, int64_t i0, int64_t i1,
                     int64_t jl, int64_t jh, int64_t kl, int64_t kh, int64_t src_lo, int64_t src_hi, Track t,
                     cudaStream_t s, int64_t* launches) {
    if (i1 <= i0 || jh <= jl || kh <= kl) return cudaSuccess;
    if (n2 % 4 != 0 || (reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) % 16 != 0 ||
        n0 >= (1ll << 31) || n1 >= (1ll << 31) || n2 >= (1ll << 31))
        return cudaErrorNotSupported;
    // the tensor map covers only the planes of src's allocation ([src_lo, src_hi) elements), so
    // the TMA unit never addresses memory outside it; plane coordinates are relative to plane_lo
    const int64_t pl = n1 * n2;
    const int64_t plane_lo = (src_lo + pl - 1) / pl, plane_hi = src_hi / pl;
    if (i0 - 1 < plane_lo || i1 + 1 > plane_hi) return cudaErrorInvalidValue;
    CUtensorMap map;
    cuuint64_t dims[3] = {(cuuint64_t)n2, (cuuint64_t)n1, (cuuint64_t)(plane_hi - plane_lo)};
    cuuint64_t strides[2] = {(cuuint64_t)n2 * 4, (cuuint64_t)n1 * n2 * 4};
    cuuint32_t box[3] = {BOXK, 18, 1};  // 16 rows + 2 halo rows
    cuuint32_t es[3] = {1, 1, 1};
    if (!tma_encode_tiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(src) + plane_lo * pl, dims,
                          strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE))
        return cudaErrorNotSupported;
    // 16 rows x 32 planes per CTA; 8 stages (more bytes in flight per SM, 2 CTAs per SM) when the
    // grid is at least 16 waves of them, else 4 stages (5 CTAs per SM, shorter tail); the other
    // tile shapes measured (32-row tiles, 64-plane segments, 6 stages) were slower
    // (profiles/r01/f2_variants.jsonl)
    const int64_t ctas = ((kh - (kl / 4) * 4 + TK - 1) / TK) * ((jh - jl + 15) / 16) * ((i1 - i0 + 31) / 32);
    if (ctas >= 16 * 2 * 148) return launch3d<16, 32, 8>(map, dst, n1, n2, i0, i1, jl, jh, kl, kh, plane_lo, t, s, launches);
    return launch3d<16, 32>(map, dst, n1, n2, i0, i1, jl, jh, kl, kh, plane_lo, t, s, launches);
}

}  // namespace k
}  // namespace accmg
