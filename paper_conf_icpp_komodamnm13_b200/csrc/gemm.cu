// Loop body: dense matmul C = A.B (config C3; the paper's "linear algebra" class of
// data-parallel loops, L72), bf16 inputs, fp32 accumulation, over one partition's rows [m0, m1).
// The parallel loop runs over (i, j) with the k-loop inside each task; rows of A and
// C are the partition's declared windows, B is replicated.
//
// This is a real contraction, so it runs on the 5th-generation tensor cores:
//   * persistent kernel, clusters of two CTAs (one CTA per SM), 128 x 256 output tiles per CTA (the
//     last n-block may be partial: N % 8 == 0), K-steps of 64; the two CTAs of a cluster take
//     vertically adjacent tiles of the same n-block (a pair tile: 2 m-blocks x 1 n-block);
//   * warp 0 = TMA producer: its A tile [128 rows][64 k] (K-major) and half of the shared B tile
//     [64 k][256 n] (N-major, two of its four 64-column boxes) multicast into both CTAs, all
//     128-byte swizzled, into a 4-stage smem ring guarded by full/empty mbarriers (a stage's empty
//     barrier counts both CTAs' MMA commits: the peer writes into it too);
//   * warp 1 = MMA issuer: one elected thread issues tcgen05.mma.cta_group::1.kind::f16
//     (M=128, N=256, K=16; A K-major, B MN-major via the instruction descriptor) accumulating in
//     TMEM; tcgen05.commit frees smem stages and signals the epilogue;
//   * warps 2-5 = epilogue: tcgen05.ld (32 lanes x 32 columns per warp and step) -> registers ->
//     128-bit global stores; two TMEM accumulators (2 x 256 columns) overlap the epilogue of tile t
//     with the MMAs of tile t+1.
// The k order of every output element is fixed (ascending 64-blocks, no split-K), so the result
// does not depend on the partition count (reading W9).
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdlib>

#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"

namespace accmg {
namespace k {
namespace {

constexpr int BM = 128, BN = 256, BK = 64;
constexpr int kStages = 4;
constexpr int kABytes = BM * BK * 2;            // 16 KiB
constexpr int kBBytes = BK * BN * 2;            // 32 KiB
constexpr int kStageBytes = kABytes + kBBytes;  // 48 KiB
constexpr int kThreads = 192;                   // 6 warps
constexpr int kTmemCols = 512;                  // 2 accumulators x 256 fp32 columns
constexpr int kGroupM = 8;                      // tile raster: 8 pair tiles (16 m-blocks) per group

using dev::mbar_arrive;
using dev::mbar_expect_tx;
using dev::mbar_init;
using dev::mbar_wait;
using dev::smem_u32;
using dev::tma_load_2d;

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tc_mma(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}

// smem matrix descriptor (tcgen05): start address, LBO, SBO in 16-byte units; version 1 (sm_100);
// layout type 2 = 128-byte swizzle.
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}

// instruction descriptor: D f32, A/B bf16, A K-major, B MN-major, N = 256, M = 128
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
                            ((uint32_t)(BM >> 4) << 24);

// Tile raster: groups of `gm_` m-blocks (here: m-block pairs) swept across all n-blocks, so the
// tiles resident at once cover a patch of C (16 m-blocks x 9.25 n-blocks: 2048 rows x 2368
// columns) and share A row-blocks / B column-blocks through L2. Measured at C3 (32768^3, same-box
// interleaved rounds; profiles/r02/experiments/gemm_raster_ab.txt, gemm_multicast_ab.txt):
// single-CTA kernel (no multicast), groups of 8 / 16 / 24 / 32 / 40 / 48 / 64 m-blocks -> 1463 /
// 1468-1478 / 1455 / 1498-1509 / 1490 / 1396-1413 / 1418-1424 TFLOP/s; this kernel with groups of
// 4 / 8 / 12 / 16 / 32 pairs -> 1376-1379 / 1497-1525 / 1494-1496 / 1468-1473 / 1238-1282 (the
// single-CTA kernel with 32 m-blocks at 1360-1405 on that box).
__device__ __forceinline__ void tile_coords(int64_t t, int num_m, int num_n, int& mb, int& nb, int gm_ = kGroupM) {
    const int64_t per_group = (int64_t)gm_ * num_n;
    const int64_t g = t / per_group;
    const int64_t r = t % per_group;
    const int gm = (int)(g * gm_);
    const int rows_in_group = (num_m - gm) < gm_ ? (num_m - gm) : gm_;
    mb = gm + (int)(r % rows_in_group);
    nb = (int)(r / rows_in_group);
}

// ---- the kernel: the two CTAs of a cluster compute vertically adjacent 128 x 256 tiles of the same
// n-block and share its B tile: CTA r loads B columns [128 r, 128 r + 128) of each k-step with a
// TMA multicast into both CTAs' shared memory (L2 -> SM traffic per CTA and stage 48 -> 32 KiB,
// which the power-capped chip turns into clock: +8-10 % over the single-CTA kernel); each CTA
// issues its own tcgen05.mma.cta_group::1 (M = 128, N = 256). A stage is refilled only after both
// CTAs' MMAs have read it: every MMA commit arrives on the stage's empty barrier of both CTAs.
// (A 2-SM cta_group::2 kernel, M = 256, and clusters of four sharing A as well as B measured
// slower: profiles/r02/experiments/README.md.)
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void tma_load_2d_mc(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1,
                                               uint16_t mask) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(
            smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "h"(mask)
        : "memory");
}
__device__ __forceinline__ void tc_commit_mc1(uint64_t* bar, uint16_t mask) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                     smem_u32(bar)),
                 "h"(mask)
                 : "memory");
}

__global__ void __launch_bounds__(kThreads, 1)
gemm_kernel(const __grid_constant__ CUtensorMap map_a, const __grid_constant__ CUtensorMap map_b,
               float* __restrict__ C, int64_t N, int64_t K, int64_t m0, int64_t m1, int64_t row_lo) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char* smem = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + kStages * kStageBytes);
    uint64_t* empty = full + kStages;
    uint64_t* tfull = empty + kStages;
    uint64_t* tempty = tfull + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t rank = cluster_rank();
    const int num_m = (int)((m1 - m0 + BM - 1) / BM);
    const int num_mp = (num_m + 1) / 2;  // m-block pairs
    const int num_n = (int)((N + BN - 1) / BN);
    const int64_t num_tiles = (int64_t)num_mp * num_n;
    const int nk = (int)(K / BK);
    const int64_t cl = blockIdx.x >> 1, ncl = gridDim.x >> 1;

    if (warp == 0 && lane == 0) {
        for (int s = 0; s < kStages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 2); }
        for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], 128); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_a)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_b)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(kTmemCols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    cluster_sync_all();  // both CTAs' barriers are initialised before any multicast reaches them
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            for (int64_t t = cl; t < num_tiles; t += ncl) {
                int mp, nb;
                tile_coords(t, num_mp, num_n, mp, nb);
                const int row = (int)(m0 + (int64_t)(2 * mp + (int)rank) * BM);
                const int col = nb * BN + 128 * (int)rank;
                for (int kb = 0; kb < nk; ++kb) {
                    mbar_wait(&empty[stage], phase ^ 1);
                    unsigned char* sa = smem + stage * kStageBytes;
                    unsigned char* sb = sa + kABytes;
                    mbar_expect_tx(&full[stage], kStageBytes);  // own A + both halves of B
                    tma_load_2d(&map_a, &full[stage], sa, kb * BK, row - (int)row_lo);
#pragma unroll
                    for (int j = 0; j < 2; ++j)
                        tma_load_2d_mc(&map_b, &full[stage], sb + (2 * rank + j) * (BK * 128), col + 64 * j, kb * BK,
                                       (uint16_t)0x3);
                    if (++stage == kStages) { stage = 0; phase ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        int stage = 0;
        uint32_t phase = 0;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int64_t t = cl; t < num_tiles; t += ncl) {
            mbar_wait(&tempty[acc], acc_phase ^ 1);
            tc_fence_after();
            const uint32_t d = tmem + (uint32_t)(acc * BN);
            for (int kb = 0; kb < nk; ++kb) {
                mbar_wait(&full[stage], phase);
                tc_fence_after();
                if (lane == 0) {
                    const uint32_t sa = smem_u32(smem + stage * kStageBytes);
                    const uint32_t sb = sa + kABytes;
#pragma unroll
                    for (int k = 0; k < BK / 16; ++k) {
                        const uint64_t da = sdesc(sa + k * 32, 16, 1024);
                        const uint64_t db = sdesc(sb + k * 2048, BK * 128, 1024);
                        tc_mma(d, da, db, kIdesc, (kb | k) ? 1u : 0u);
                    }
                    tc_commit_mc1(&empty[stage], (uint16_t)0x3);
                }
                __syncwarp();
                if (++stage == kStages) { stage = 0; phase ^= 1; }
            }
            if (lane == 0) tc_commit(&tfull[acc]);
            __syncwarp();
            if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        }
    } else {
        const int q = warp & 3;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int64_t t = cl; t < num_tiles; t += ncl) {
            int mp, nb;
            tile_coords(t, num_mp, num_n, mp, nb);
            mbar_wait(&tfull[acc], acc_phase);
            tc_fence_after();
            const int64_t row = m0 + (int64_t)(2 * mp + (int)rank) * BM + q * 32 + lane;
            float* crow = C + row * N + (int64_t)nb * BN;
            const bool ok = row < m1;
            const int ncols = (int)((N - (int64_t)nb * BN) < BN ? (N - (int64_t)nb * BN) : BN);
#pragma unroll 1
            for (int c = 0; c < BN / 32; ++c) {
                uint32_t v[32];
                const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * BN + c * 32);
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
                    "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                    : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                      "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                      "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                      "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                      "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
                    : "r"(taddr));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                if (ok) {
                    float4* dst = reinterpret_cast<float4*>(crow + c * 32);
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        if (c * 32 + 4 * j < ncols)
                            dst[j] = make_float4(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]),
                                                 __uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3]));
                }
            }
            tc_fence_before();
            mbar_arrive(&tempty[acc]);
            if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        }
    }
    tc_fence_before();
    cluster_sync_all();  // no multicast or remote arrive may target a CTA that has exited
    tc_fence_after();
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

bool make_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t row_bytes, uint32_t box_in,
              uint32_t box_out) {
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {row_bytes};
    cuuint32_t box[2] = {box_in, box_out};
    cuuint32_t es[2] = {1, 1};
    return tma_encode_tiled(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

}  // namespace

cudaError_t gemm_bf16(const uint16_t* A, const uint16_t* B, float* C, int64_t M, int64_t N, int64_t K, int64_t m0,
                      int64_t m1, int64_t a_lo, cudaStream_t s, int64_t* launches) {
    (void)M;
    if (m1 <= m0) return cudaSuccess;
    // N % 8: B rows are 16-byte multiples for the TMA and C rows take 128-bit stores
    if (N % 8 != 0 || K % BK != 0 || K >= (1ll << 31) || N >= (1ll << 31) || m1 >= (1ll << 31))
        return cudaErrorNotSupported;
    // A's map starts at the first whole row of its allocation, so the TMA unit never addresses
    // rows outside it (row coordinates are relative to row_lo)
    const int64_t row_lo = (a_lo + K - 1) / K;
    if (m0 < row_lo) return cudaErrorInvalidValue;
    CUtensorMap ma, mb;
    if (!make_map(&ma, A + row_lo * K, (uint64_t)K, (uint64_t)(m1 - row_lo), (uint64_t)K * 2, BK, BM))
        return cudaErrorNotSupported;
    if (!make_map(&mb, B, (uint64_t)N, (uint64_t)K, (uint64_t)N * 2, 64, BK)) return cudaErrorNotSupported;
    const int sms = sm_count_cached();
    const size_t smem = 1024 + (size_t)kStages * kStageBytes + 256;
    cudaError_t e = kernel_prep(gemm_kernel, kThreads, smem);
    if (e != cudaSuccess) return e;
    // one cluster of two CTAs per SM pair, persistent over the pair tiles (2 m-blocks x 1 n-block);
    // no more clusters than can be resident at once (a GPC with an odd SM count leaves one out)
    const int64_t ptiles = ((m1 - m0 + 2 * BM - 1) / (2 * BM)) * ((N + BN - 1) / BN);
    int64_t ncl = sms / 2;
    static int max_cl = 0;
    if (!max_cl) {
        cudaLaunchConfig_t q{};
        q.gridDim = dim3((unsigned)(2 * ncl));
        q.blockDim = dim3(kThreads);
        q.dynamicSmemBytes = smem;
        cudaLaunchAttribute qa[1];
        qa[0].id = cudaLaunchAttributeClusterDimension;
        qa[0].val.clusterDim.x = 2;
        qa[0].val.clusterDim.y = 1;
        qa[0].val.clusterDim.z = 1;
        q.attrs = qa;
        q.numAttrs = 1;
        int n = 0;
        max_cl = (cudaOccupancyMaxActiveClusters(&n, gemm_kernel, &q) == cudaSuccess && n > 0) ? n : (int)ncl;
        (void)cudaGetLastError();
    }
    if (ncl > max_cl) ncl = max_cl;
    if (ptiles < ncl) ncl = ptiles;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)(2 * ncl));
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, gemm_kernel, ma, mb, C, N, K, m0, m1, row_lo);
    if (e != cudaSuccess) return e;
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
