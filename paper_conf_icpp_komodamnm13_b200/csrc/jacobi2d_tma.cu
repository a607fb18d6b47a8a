// Loop body variant: 2-D 5-point Jacobi with TMA-staged shared-memory tiles (impl = 2).
//
// Same operation and rounding as jacobi.cu. Each CTA owns a 128-column strip and a segment of
// tpc x 32 rows (tpc <= 8, chosen per launch to balance the waves); one thread streams
// (32 + 2) x 136-float tiles (rows with their halo rows, columns with 4 halo columns each side)
// through a 4-stage ring with cp.async.bulk.tensor.2d
// completing on mbarriers; 8 warps compute 4 rows x 4 columns per lane from shared memory
// (horizontal neighbours by shuffle) and store 128-bit vectors of interior points. The halo rows
// of a tile are the previous / next tile's edge rows, so their second read hits L2.
// The default body (measured faster than the register-marching kernel, impl = 1: profiles/ and
// DESIGN.md). Write tracking (undeclared dst) runs once per CTA after its stores: mark_rect sets
// the words of its (32 tpc)-row x 128-column rectangle (plain stores for owned words, atomicOr on words
// shared with the neighbouring strips) and the rows' chunk bits.
#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"
#include "track.cuh"

namespace accmg {
namespace k {
namespace {

constexpr int TK = 128;
constexpr int RB = 32;             // rows computed per tile
constexpr int BOXK = TK + 8;
constexpr int BOXR = RB + 2;
constexpr int kStages = 4;
constexpr int kMaxTiles = 8;       // tiles per CTA (up to 256 rows; chosen per launch)
constexpr uint32_t kTileBytes = BOXK * BOXR * 4;
constexpr int kStageFloats = ((kTileBytes + 127) / 128) * 32;  // 128-byte aligned stages

__device__ __forceinline__ float st5(float n, float s, float w, float e) {
    return __fmul_rn(__fadd_rn(__fadd_rn(n, s), __fadd_rn(w, e)), 0.25f);
}

template <bool TRACK>
__global__ void __launch_bounds__(256)
jacobi2d_tma_k(const __grid_constant__ CUtensorMap map, float* __restrict__ dst, int64_t cols, int64_t r0, int64_t r1,
               int64_t c0, int64_t c1, int64_t cbase, int64_t row_lo, int tpc, Track t, const HaloPush push) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    float* tiles = reinterpret_cast<float*>(smem_raw);
    __shared__ __align__(8) uint64_t bar[kStages];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t k0 = cbase + (int64_t)blockIdx.x * TK;
    const int64_t rs = r0 + (int64_t)blockIdx.y * (RB * tpc);
    if (rs >= r1) return;
    const int ntiles = (int)((((r1 - rs) < RB * tpc ? (r1 - rs) : RB * tpc) + RB - 1) / RB);
    // programmatic dependent launch: the next loop's body may be scheduled while this grid drains
    // (its CTAs wait here, after their setup, until this grid has completed and flushed), so the
    // launch latency between consecutive sweeps overlaps the tail of the previous one
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) dev::mbar_init(&bar[s], 1);
        dev::mbar_fence_init();
        dev::tma_prefetch_desc(&map);
    }
    asm volatile("griddepcontrol.wait;" ::: "memory");  // src (and dst) are the previous loop's arrays
    if (tid == 0) {
        for (int m = 0; m < kStages && m < ntiles; ++m) {
            dev::mbar_expect_tx(&bar[m], kTileBytes);
            dev::tma_load_2d(&map, &bar[m], tiles + m * kStageFloats, (int)(k0 - 4), (int)(rs + RB * m - 1 - row_lo));
        }
    }
    __syncthreads();
    const int64_t k = k0 + 4 * lane;
    unsigned nib = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c) nib |= (k + c >= c0 && k + c < c1) ? (1u << c) : 0u;
    const bool full = nib == 0xFu;
    const int col = 4 + 4 * lane;
    for (int m = 0; m < ntiles; ++m) {
        const int st = m % kStages;
        dev::mbar_wait(&bar[st], (uint32_t)((m / kStages) & 1));
        const float* T = tiles + st * kStageFloats;
        // rows 4*warp .. 4*warp+3 of the tile (tile row index = row + 1)
        float4 R[6];
#pragma unroll
        for (int q = 0; q < 6; ++q) R[q] = *reinterpret_cast<const float4*>(T + (4 * warp + q) * BOXK + col);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int64_t row = rs + (int64_t)RB * m + 4 * warp + q;
            const float4 C = R[q + 1], N = R[q], S = R[q + 2];
            float w = __shfl_up_sync(dev::kFull, C.w, 1);
            float e = __shfl_down_sync(dev::kFull, C.x, 1);
            if (lane == 0) w = T[(4 * warp + q + 1) * BOXK + col - 1];
            if (lane == 31) e = T[(4 * warp + q + 1) * BOXK + col + 4];
            if (row < r1) {  // warp-uniform
                float o[4];
                o[0] = st5(N.x, S.x, w, C.y);
                o[1] = st5(N.y, S.y, C.x, C.z);
                o[2] = st5(N.z, S.z, C.y, C.w);
                o[3] = st5(N.w, S.w, C.z, e);
                float* out = dst + row * cols + k;
                if (full) {
                    *reinterpret_cast<float4*>(out) = make_float4(o[0], o[1], o[2], o[3]);
                } else {
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (nib & (1u << c)) out[c] = o[c];
                }
#pragma unroll
                for (int pi = 0; pi < kMaxPush; ++pi) {  // predicted readers' copies (static indices:
                    // the parameter block stays in constant space)
                    if (pi >= push.n || row < push.lo[pi] || row >= push.hi[pi]) continue;  // warp-uniform
                    float* pout = push.dst[pi] + row * cols + k;
                    if (full) {
                        *reinterpret_cast<float4*>(pout) = make_float4(o[0], o[1], o[2], o[3]);
                    } else {
#pragma unroll
                        for (int c = 0; c < 4; ++c)
                            if (nib & (1u << c)) pout[c] = o[c];
                    }
                }
            }
        }
        __syncthreads();  // every thread is done with stage st
        if (tid == 0 && m + kStages < ntiles) {
            const int mn = m + kStages;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            dev::mbar_expect_tx(&bar[st], kTileBytes);
            dev::tma_load_2d(&map, &bar[st], tiles + st * kStageFloats, (int)(k0 - 4),
                             (int)(rs + RB * mn - 1 - row_lo));
        }
    }
    if constexpr (TRACK) {  // dirty bits of the CTA's rectangle, once, after its stores
        const int64_t re = rs + (int64_t)RB * tpc < r1 ? rs + (int64_t)RB * tpc : r1;
        dev::mark_rect(t.l1, t.l2, t.l2_shift, rs, re, cols, k0 > c0 ? k0 : c0, k0 + TK < c1 ? k0 + TK : c1, tid, 256);
    }
}

}  // namespace

cudaError_t jacobi2d_tma(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1, int64_t c0,
                         int64_t c1, int64_t src_lo, int64_t src_hi, Track t, cudaStream_t s, int64_t* launches,
                         const HaloPush& push) {
    (void)rows;
    if (r1 <= r0 || c1 <= c0) return cudaSuccess;
    uintptr_t align = reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst);
    for (int i = 0; i < push.n; ++i) align |= reinterpret_cast<uintptr_t>(push.dst[i]);  // 128-bit pushes too
    if (cols % 4 != 0 || align % 16 != 0 || cols >= (1ll << 31)) return cudaErrorNotSupported;
    // the map covers only the whole rows of src's allocation (row coordinates relative to row_lo)
    const int64_t row_lo = (src_lo + cols - 1) / cols, row_hi = src_hi / cols;
    if (r0 - 1 < row_lo || r1 + 1 > row_hi) return cudaErrorInvalidValue;
    CUtensorMap map;
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)(row_hi - row_lo)};
    cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
    cuuint32_t box[2] = {BOXK, BOXR};
    cuuint32_t es[2] = {1, 1};
    if (!tma_encode_tiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(src) + row_lo * cols, dims,
                          strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE))
        return cudaErrorNotSupported;
    const int64_t cbase = (c0 / 4) * 4;
    const size_t smem = (size_t)kStages * kStageFloats * 4;
    auto kern = t.l1 ? jacobi2d_tma_k<true> : jacobi2d_tma_k<false>;
    int per_sm = 1;
    cudaError_t e = kernel_prep(kern, 256, smem, &per_sm);
    if (e != cudaSuccess) return e;
    // rows per CTA (32 x tpc): the grid runs in waves of (resident CTAs per SM x SMs); pick tpc so
    // that waves x (rows + 2 halo rows) per CTA is smallest -- a 4095-row partition (C2 at P = 8)
    // runs 10 waves of 256-row CTAs with the last one 23 % full, but 15 full waves of 160 rows
    const int nsm = sm_count_cached();
    const int64_t strips = (c1 - cbase + TK - 1) / TK, slots = (int64_t)nsm * (per_sm > 0 ? per_sm : 1);
    int tpc = kMaxTiles;
    int64_t best = -1;
    for (int q = kMaxTiles; q >= 2; --q) {
        const int64_t segs = (r1 - r0 + RB * q - 1) / (RB * q);
        const int64_t cost = (strips * segs + slots - 1) / slots * (RB * q + 2);
        if (best < 0 || cost * 100 < best * 98) {  // smaller tiles only for a >= 2 % gain
            best = cost;
            tpc = q;
        }
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)strips, (unsigned)((r1 - r0 + RB * tpc - 1) / (RB * tpc)));
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, kern, map, dst, cols, r0, r1, c0, c1, cbase, row_lo, tpc, t, push);
    if (e != cudaSuccess) return e;
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
