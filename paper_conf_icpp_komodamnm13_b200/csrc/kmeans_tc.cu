// k-means assignment loop + reductiontoarray (config C4) on the tcgen05 tensor cores, bit-exact with
// the scalar loop of the paper's KMEANS (Table II; reading KM in DESIGN.md):
//
//   D_f(p, c) = fmaf chain over j of (x[p][j] - cen[c][j])^2,   member[p] = lowest c minimising D_f,
//   sums[member[p]][j] += x[p][j] * 2^shift (exact int64),        counts[member[p]] += 1.
//
// Both halves of the loop are dense contractions once written as matrices:
//   * distances: argmin_c D = argmax_c V, V(p, c) = x.c - |c|^2/2 — an (n x 16) by (16 x k) product.
//     A = [x0 | x0 | x1 | 1 1 1], B = [c0 | c1 | c0 | h0 h1 h2] (bf16 pieces: x = x0 + x1 + e with
//     |e| <= 2^-16 |x|, -|c|^2/2 = h0 + h1 + h2), four tcgen05.mma.kind::f16 (K = 64) give
//     v = x0.c0 + x0.c1 + x1.c0 - |c|^2/2 in TMEM, fp32, one 128-column half of the centroids per
//     accumulator; each half is handed back to the MMA warp as soon as the epilogue has read it,
//     so the next tile's MMAs of that half overlap the epilogue's remaining work;
//   * reductiontoarray: sums[c][(j, b)] = sum_p onehot[c][p] * byte_b(x[p][j] * 2^shift + 2^31) and
//     counts[c] = sum_p onehot[c][p] * 1 — tcgen05.mma.kind::i8 (u8 x u8 -> s32, exact) with
//     A = the one-hot assignment matrix [128 clusters][128 points] and B = the points' fixed-point
//     byte planes [80 rows][128 points]; the s32 accumulators stay in TMEM across all the CTA's
//     tiles and are read once at the end (no atomics per point).
// Exactness of the assignment: every c with v(c) >= vmax - T is a candidate and is re-evaluated
// with the exact fmaf chain (ascending c, strict <), T a rigorous bound of the filter error:
// with Cinf = max |cen|, C2 = max |c|^2, L1 = sum |x_j|, Q = sum x_j^2,
//   |v - V| <= E := 2^-11 (L1 Cinf + C2)  (split 3.1*2^-16 L1 Cinf, hn split 2^-24 C2, fp32
//   accumulation of 51 products <= 51*2^-23 (L1 Cinf + C2): >= 6x slack),
//   T = 2E + 2^-16 Dhat, Dhat = Q (1 + 2^-17) - 2 vmax + 2E >= D(p, c^) (c^ = argmax v).
// A non-candidate c has V(c^) - V(c) > 2^-16 Dhat, so D(c) - D(c^) > 2^-15 D(c^) >= eps (D(c) +
// D(c^)) with the fmaf chain's relative error eps <= 18 * 2^-24 (non-negative terms): D_f(c) >
// D_f(c^), it can neither win nor tie. Inputs are on the 2^-shift grid (W4). CPU pins of this
// reading: tests/test_kmeans_filter_bound.py.
//
// Warp roles (one CTA per SM, persistent over 128-point tiles):
//   w0 producer: TMA load (64-byte swizzle) of the tile's fp32 rows (8 KiB) into an mbarrier ring;
//   w1 MMA issuer (one thread): distance MMAs of tile i, then the reduction MMAs of tile i-1;
//   w2-5 converters (one point per thread): bf16 pieces of x into the distance A operand, the
//        fixed-point bytes into the reduction B operand, the 2^-shift grid check, the point's
//        bound terms E and Q(1 + 2^-17) + 2E for the epilogue;
//   w6-9 epilogue (one point per thread = TMEM lane): pass 1 = maxima of 4-column groups (3-input
//        FMNMX) over all k columns, then a candidate-group mask (sign bits of thr - max, packed
//        FSUB2, funnel-shifted), the exact re-check of the candidate groups (packed FADD2 / FFMA2,
//        each lane rounding like the scalar op), member[p] and the point's one-hot byte.
// Same-box A/B measurements of the alternatives tried: profiles/r01/kmeans_tc.log.
#include <cuda_bf16.h>

#include <cstdlib>

#include "kernels.h"
#include "tma_dev.cuh"
#include "tma_host.h"

namespace accmg {
namespace k {
namespace {

using dev::mbar_arrive;
using dev::mbar_expect_tx;
using dev::mbar_init;
using dev::mbar_wait;
using dev::smem_u32;

constexpr int TM = 128;                 // points per tile (distance MMA M, reduction MMA K)
constexpr int KMAX = 256;               // centroids
constexpr int XS = 4;                   // fp32 point-tile stages
constexpr int AS = 2;                   // distance A operand stages (freed by the distance MMAs)
constexpr int BS = 4;                   // reduction B operand stages (freed by the reduction MMAs)
constexpr int OS = 2;                   // one-hot stages
constexpr int kRows = 80;               // reduction B rows: 16 dims x 4 bytes, counts, 15 zero
constexpr int kXBytes = TM * 64;        // 8 KiB
constexpr int kADBytes = TM * 128;      // 16 KiB
constexpr int kABBytes = kRows * 128;   // 10 KiB
constexpr int kOHBytes = KMAX * 128;    // 32 KiB (two 128-cluster halves)
constexpr int kThreadsTC = 320;
constexpr int kTmemCols = 512;
constexpr uint32_t kColSum = 256;       // reduction accumulators: half h at 256 + 80 h

constexpr int OFF_AD = 0;
constexpr int OFF_AB = OFF_AD + AS * kADBytes;
constexpr int OFF_BD = OFF_AB + BS * kABBytes;
constexpr int OFF_OH = OFF_BD + KMAX * 128;
constexpr int OFF_X = OFF_OH + OS * kOHBytes;
// re-check copy of the centroids, negated, for packed pairs: group G = centroids 4G..4G+3 at
// G * kGrpBytes (16 B of padding per group spreads the lanes' groups over the banks), pair P of
// the group at +128 P, dims (j, j+1) of both centroids of the pair at +8 j: one LDS.128
constexpr int kGrpBytes = 272;
constexpr int OFF_PC = OFF_X + XS * kXBytes;
constexpr int OFF_BAR = OFF_PC + (KMAX / 4) * kGrpBytes;
constexpr int kMaxQ = 8;                // distance accumulator column groups (>= KMAX / QW)
constexpr int kNumBars = 2 * XS + 2 * AS + BS + 2 * kMaxQ + 2 * OS + 1;
constexpr int OFF_MISC = OFF_BAR + kNumBars * 8;    // tmem slot, Cinf bits, C2 bits
constexpr int OFF_EQ = OFF_MISC + 16;               // float2 [BS][TM]: the point's E and Q (1 + 2^-17) + 2E
constexpr int kSmemTC = OFF_EQ + BS * TM * 8 + 1024;  // + alignment slack
static_assert(OFF_AB % 1024 == 0 && OFF_BD % 1024 == 0 && OFF_OH % 1024 == 0 && OFF_X % 1024 == 0, "align");
static_assert(kSmemTC <= 227 * 1024, "smem");

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mma_f16(uint32_t d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void mma_i8(uint32_t d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}
// K-major operand, 128-byte swizzle: rows of 128 B, 8-row atoms 1024 B apart (SBO), version 1.
__device__ __forceinline__ uint64_t sdesc_sw128(uint32_t saddr) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)(16 >> 4) << 16;
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}
// byte offset of element k (byte k) of row m in a 128-byte-swizzled K-major operand
__device__ __forceinline__ uint32_t sw_off(uint32_t m, uint32_t kbyte) {
    return m * 128u + ((((kbyte >> 4) ^ (m & 7u)) << 4) | (kbyte & 15u));
}
// wait with a suspend-time hint: a warp that waits for a free stage sleeps instead of spinning on
// issue slots the converter / epilogue warps of its SM sub-partition need
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAITS_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra WAITS_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity), "r"(20000u)
        : "memory");
}
__device__ __forceinline__ void sts_u8(uint32_t addr, uint32_t v) {
    asm volatile("st.shared.u8 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_v4(uint32_t addr, uint4 v) {
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}
__device__ __forceinline__ float4 lds_f4(uint32_t addr) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr));
    return v;
}

__device__ __forceinline__ uint32_t bf2(float a, float b) {  // bf16_rn(a) | bf16_rn(b) << 16
    const __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<const uint32_t*>(&h);
}
// 8 values -> two 16-byte chunks of hi pieces and of lo pieces (x = hi + lo + e)
__device__ __forceinline__ void split8(const float* x, uint4& hi, uint4& lo) {
    uint32_t h[4], l[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        h[i] = bf2(x[2 * i], x[2 * i + 1]);
        const float ha = __uint_as_float(h[i] << 16), hb = __uint_as_float(h[i] & 0xFFFF0000u);
        l[i] = bf2(x[2 * i] - ha, x[2 * i + 1] - hb);
    }
    hi = make_uint4(h[0], h[1], h[2], h[3]);
    lo = make_uint4(l[0], l[1], l[2], l[3]);
}

template <int N>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&r)[N]);
template <>
__device__ __forceinline__ void tmem_ld<32>(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
          "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
          "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
template <>
__device__ __forceinline__ void tmem_ld<16>(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ uint64_t pk2(float a, float b) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ void upk2(uint64_t v, float& a, float& b) {
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
// packed fp32x2 (PTX add/fma .f32x2): each lane rounds exactly like the scalar add.rn / fma.rn
__device__ __forceinline__ uint64_t add2(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ uint64_t sub2(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ uint64_t fma2(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}

__device__ __forceinline__ float max3(float a, float b, float c) {
    float d;
    asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
    return d;
}

__device__ __forceinline__ float next_below(float a) {
    if (a == 0.f) return -0x1p-149f;
    const int b = __float_as_int(a);
    return __int_as_float(a > 0.f ? b - 1 : b + 1);
}

// QW: width (centroid columns) of each distance accumulator; each has its own full / empty
// barriers, so the MMAs of the next tile refill a group as soon as the epilogue has read it
template <int QW>
__global__ void __launch_bounds__(kThreadsTC, 1)
assign_tc(const __grid_constant__ CUtensorMap xmap, const float* __restrict__ cen, int32_t* __restrict__ member,
          int64_t* __restrict__ sums, int64_t* __restrict__ counts, int64_t p0, int64_t p1, int kc, int npad,
          int shift, int* err) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    // aligned base inside the shared window (address arithmetic on smem_raw keeps the state space)
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t pad = ((raw + 1023u) & ~1023u) - raw;
    unsigned char* smem = smem_raw + pad;
    const uint32_t sbase = raw + pad;
    const uint32_t sAD = sbase + OFF_AD, sAB = sbase + OFF_AB, sBD = sbase + OFF_BD, sOH = sbase + OFF_OH;
    const uint32_t sX = sbase + OFF_X, sPC = sbase + OFF_PC;
    uint64_t* xfull = reinterpret_cast<uint64_t*>(smem + OFF_BAR);
    uint64_t* xempty = xfull + XS;
    uint64_t* afull = xempty + XS;
    uint64_t* aempty = afull + AS;
    uint64_t* bempty = aempty + AS;
    uint64_t* dfull = bempty + BS;
    uint64_t* dempty = dfull + kMaxQ;
    uint64_t* ofull = dempty + kMaxQ;
    uint64_t* oempty = ofull + OS;
    uint64_t* sdone = oempty + OS;
    uint32_t* misc = reinterpret_cast<uint32_t*>(smem + OFF_MISC);  // [0] tmem, [1] Cinf bits, [2] C2 bits

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t ntiles = (p1 - p0 + TM - 1) / TM;
    const int64_t nt = blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    const uint32_t nt32 = (uint32_t)nt;
    const int nh = (npad + 127) / 128;  // 128-centroid halves (reduction)
    constexpr int NQ = KMAX / QW;       // distance accumulator groups
    const int nq = (npad + QW - 1) / QW;

    // ---- setup: constant operand parts, centroids, bounds, barriers, TMEM
    if (tid == 0) { misc[1] = 0u; misc[2] = 0u; }
    for (int i = tid; i < npad * 16; i += kThreadsTC) {
        const int c = i >> 4, j = i & 15;
        const float v = c < kc ? -cen[i] : 0.f;
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sPC + (c >> 2) * kGrpBytes + ((c >> 1) & 1) * 128 + j * 8 +
                                                    (c & 1) * 4),
                     "f"(v)
                     : "memory");
    }
    for (uint32_t i = tid; i < OS * kOHBytes / 16; i += kThreadsTC) sts_v4(sOH + i * 16, make_uint4(0, 0, 0, 0));
    for (int i = tid; i < AS * TM; i += kThreadsTC) {  // distance A, slice 3 = [1 1 1 0 ...]
        const uint32_t base = sAD + (i / TM) * kADBytes, r = i % TM;
        sts_v4(base + sw_off(r, 96), make_uint4(0x3F803F80u, 0x00003F80u, 0, 0));
        sts_v4(base + sw_off(r, 112), make_uint4(0, 0, 0, 0));
    }
    for (int i = tid; i < BS * 16 * 8; i += kThreadsTC) {  // reduction B rows 64 (= 1) and 65..79 (= 0)
        const int a = i / 128, row = 64 + (i % 128) / 8, ch = i % 8;
        const uint32_t v = row == 64 ? 0x01010101u : 0u;
        sts_v4(sAB + a * kABBytes + row * 128 + ch * 16, make_uint4(v, v, v, v));
    }
    if (tid == 0) {
        for (int s = 0; s < XS; ++s) { mbar_init(&xfull[s], 1); mbar_init(&xempty[s], 256); }
        for (int a = 0; a < AS; ++a) { mbar_init(&afull[a], 128); mbar_init(&aempty[a], 1); }
        for (int b = 0; b < BS; ++b) mbar_init(&bempty[b], 1);
        for (int b = 0; b < kMaxQ; ++b) { mbar_init(&dfull[b], 1); mbar_init(&dempty[b], 128); }
        for (int o = 0; o < OS; ++o) { mbar_init(&ofull[o], 128); mbar_init(&oempty[o], 1); }
        mbar_init(sdone, 1);
        dev::mbar_fence_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(misc)),
                     "r"(kTmemCols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    __syncthreads();
    for (int n = tid; n < npad; n += kThreadsTC) {  // distance B rows [c0 | c1 | c0 | h0 h1 h2 0 ...]
        float c[16];
        float q = 0.f, m = 0.f;
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            c[j] = n < kc ? cen[n * 16 + j] : 0.f;
            q = fmaf(c[j], c[j], q);
            m = fmaxf(m, fabsf(c[j]));
        }
        uint4 h0, l0, h1, l1;
        split8(c, h0, l0);
        split8(c + 8, h1, l1);
        sts_v4(sBD + sw_off(n, 0), h0);
        sts_v4(sBD + sw_off(n, 16), h1);
        sts_v4(sBD + sw_off(n, 32), l0);
        sts_v4(sBD + sw_off(n, 48), l1);
        sts_v4(sBD + sw_off(n, 64), h0);
        sts_v4(sBD + sw_off(n, 80), h1);
        uint32_t n01, n2;
        if (n < kc) {
            const float nh_ = -0.5f * q;  // exact scaling; any summation order (filter only)
            const float a0 = __bfloat162float(__float2bfloat16_rn(nh_));
            const float a1 = __bfloat162float(__float2bfloat16_rn(nh_ - a0));
            const float a2 = nh_ - a0 - a1;
            n01 = bf2(a0, a1);
            n2 = bf2(a2, 0.f);

            atomicMax(&misc[1], __float_as_uint(m));  // non-negative floats order as their bits
            atomicMax(&misc[2], __float_as_uint(q));
        } else {
            const uint4 z = make_uint4(0, 0, 0, 0);
            sts_v4(sBD + sw_off(n, 0), z);
            sts_v4(sBD + sw_off(n, 16), z);
            sts_v4(sBD + sw_off(n, 32), z);
            sts_v4(sBD + sw_off(n, 48), z);
            sts_v4(sBD + sw_off(n, 64), z);
            sts_v4(sBD + sw_off(n, 80), z);
            n01 = bf2(-0x1p100f, 0.f);  // padding centroid: v = -2^100, never a candidate
            n2 = 0u;

        }
        sts_v4(sBD + sw_off(n, 96), make_uint4(n01, n2, 0, 0));
        sts_v4(sBD + sw_off(n, 112), make_uint4(0, 0, 0, 0));
    }
    fence_async_smem();  // operands written by generic-proxy stores are read by tcgen05.mma
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = misc[0];

    if (warp == 0) {
        // ---- producer
        if (lane == 0) {
            for (uint32_t i = 0; i < nt32; ++i) {
                const uint32_t t = blockIdx.x + i * gridDim.x;
                const int s = (int)(i % XS);
                mbar_wait_sleep(&xempty[s], (uint32_t)((i / XS) & 1) ^ 1u);
                mbar_expect_tx(&xfull[s], kXBytes);  // rows past the end are zero-filled
                dev::tma_load_2d(&xmap, &xfull[s], smem + OFF_X + s * kXBytes, 0, (int)(t * TM));
            }
        }
    } else if (warp == 1) {
        // ---- MMA issuer (one thread)
        if (lane == 0) {
            const uint32_t idesc_sum = (2u << 4) | ((uint32_t)(kRows >> 3) << 17) | ((uint32_t)(TM >> 4) << 24);
            auto reduce = [&](uint32_t j) {
                const int o = (int)(j % OS);
                mbar_wait_sleep(&ofull[o], (uint32_t)((j / OS) & 1));
                tc_fence_after();
                const uint32_t b = sAB + (uint32_t)(j % BS) * kABBytes;
                for (int h = 0; h < nh; ++h)
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        mma_i8(tmem + kColSum + 80u * h, sdesc_sw128(sOH + o * kOHBytes + h * 16384 + k * 32),
                               sdesc_sw128(b + k * 32), idesc_sum, (j | k) ? 1u : 0u);
                tc_commit(&oempty[o]);
                tc_commit(&bempty[j % BS]);
            };
            for (uint32_t i = 0; i < nt32; ++i) {
                const int a = (int)(i % AS);
                mbar_wait_sleep(&afull[a], (uint32_t)((i / AS) & 1));
                for (int g = 0; g < nq; ++g) {
                    mbar_wait_sleep(&dempty[g], (uint32_t)(i & 1) ^ 1u);
                    tc_fence_after();
                    const int wq = (npad - QW * g) < QW ? (npad - QW * g) : QW;
                    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(wq >> 3) << 17) |
                                           ((uint32_t)(TM >> 4) << 24);
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        // A slices x0, x0, x1, 1 (slice 0 read twice) against B slices c0, c1, c0, h
                        mma_f16(tmem + (uint32_t)(QW * g), sdesc_sw128(sAD + a * kADBytes + (k == 1 ? 0 : k * 32)),
                                sdesc_sw128(sBD + g * QW * 128 + k * 32), idesc, k ? 1u : 0u);
                    tc_commit(&dfull[g]);
                }
                tc_commit(&aempty[a]);
                if (i >= 1) reduce(i - 1);
            }
            if (nt32 > 0) reduce(nt32 - 1);
            tc_commit(sdone);
        }
    } else if (warp < 6) {
        // ---- converters: point row r
        const int r = tid - 64;
        const float scale = (float)(1 << shift);
        const float Cinf = __uint_as_float(misc[1]);
        const float C2 = __uint_as_float(misc[2]);
        int bad = 0;
        for (uint32_t i = 0; i < nt32; ++i) {
            const int s = (int)(i % XS), a = (int)(i % AS);
            mbar_wait_sleep(&xfull[s], (uint32_t)((i / XS) & 1));
            float xv[16];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const float4 v = lds_f4(sX + s * kXBytes + r * 64 + ((j ^ ((r >> 1) & 3)) << 4));
                xv[4 * j] = v.x; xv[4 * j + 1] = v.y; xv[4 * j + 2] = v.z; xv[4 * j + 3] = v.w;
            }
            mbar_arrive(&xempty[s]);
            mbar_wait_sleep(&aempty[a], (uint32_t)((i / AS) & 1) ^ 1u);
            const int bs = (int)(i % BS);
            mbar_wait_sleep(&bempty[bs], (uint32_t)((i / BS) & 1) ^ 1u);
            uint4 h0, l0, h1, l1;
            split8(xv, h0, l0);
            split8(xv + 8, h1, l1);
            const uint32_t ad = sAD + a * kADBytes;
            // slices 0 = x0, 2 = x1 (3 = the constant ones); the MMA reads slice 0 twice
            sts_v4(ad + sw_off(r, 0), h0);
            sts_v4(ad + sw_off(r, 16), h1);
            sts_v4(ad + sw_off(r, 64), l0);
            sts_v4(ad + sw_off(r, 80), l1);
            // fixed point x * 2^shift, biased to unsigned: u = v + 2^31; byte b of dim j -> row 4j + b
            // row m = 4j + b has swizzle phase m & 7 = 4 (j & 1) + b: eight per-thread base addresses,
            // the row offset m * 128 is the store's immediate (st.shared.u8 keeps the low byte)
            const uint32_t ab = sAB + bs * kABBytes;
            uint32_t base[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) base[k] = ab + ((((uint32_t)r >> 4) ^ (uint32_t)k) << 4) + ((uint32_t)r & 15u);
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const float v = xv[j] * scale;  // exact: power-of-two scaling
                const float av = fabsf(v);
                const float m = copysignf(8388608.0f, v);
                const bool ok = av < 2147483648.0f && (av >= 8388608.0f || __fsub_rn(__fadd_rn(v, m), m) == v);
                bad |= !ok;
                const uint32_t u = (uint32_t)__float2int_rn(v) ^ 0x80000000u;
#pragma unroll
                for (int b = 0; b < 4; ++b)
                    sts_u8(base[4 * (j & 1) + b] + (uint32_t)((4 * j + b) * 128), u >> (8 * b));
            }
            {  // the filter bound's per-point terms, for the epilogue (header: E, Dhat)
                float L1 = 0.f, Q = 0.f;
#pragma unroll
                for (int j = 0; j < 16; ++j) { L1 += fabsf(xv[j]); Q = fmaf(xv[j], xv[j], Q); }
                const float E = (0x1p-11f * (L1 * Cinf + C2)) * 1.001f + 0x1p-100f;
                const float Qa = Q * (1.f + 0x1p-17f) + 2.f * E;
                asm volatile("st.shared.v2.f32 [%0], {%1, %2};" ::"r"(sbase + OFF_EQ + (bs * TM + r) * 8), "f"(E), "f"(Qa)
                             : "memory");
            }
            fence_async_smem();
            mbar_arrive(&afull[a]);
        }
        if (bad) atomicOr(err, 1);
    } else {
        // ---- epilogue: point row r = TMEM lane
        const int q = warp & 3;
        const int r = q * 32 + lane;
        int32_t pend[OS];
#pragma unroll
        for (int o = 0; o < OS; ++o) pend[o] = -1;
        for (uint32_t i = 0; i < nt32; ++i) {
            const uint32_t t = blockIdx.x + i * gridDim.x;
            const int s = (int)(i % XS);
            const uint32_t pr = t * TM + (uint32_t)r;  // row within the partition (< 2^31)
            const int64_t p = p0 + pr;
            const bool valid = pr < (uint32_t)(p1 - p0);
            mbar_wait(&xfull[s], (uint32_t)((i / XS) & 1));
            float xv[16];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const float4 v = lds_f4(sX + s * kXBytes + r * 64 + ((j ^ ((r >> 1) & 3)) << 4));
                xv[4 * j] = v.x; xv[4 * j + 1] = v.y; xv[4 * j + 2] = v.z; xv[4 * j + 3] = v.w;
            }
            mbar_arrive(&xempty[s]);
            // pass 1 over the accumulator groups: maxima of the 4-column groups (64 registers); each
            // accumulator goes back to the MMA warp as soon as it is read
            float gm[64];
#pragma unroll
            for (int qg = 0; qg < NQ; ++qg) {
                if (qg < nq) {
                    mbar_wait_sleep(&dfull[qg], (uint32_t)(i & 1));
                    tc_fence_after();
                }
                const int ncq = qg < nq ? (((npad - QW * qg) < QW ? (npad - QW * qg) : QW) / 32) : 0;
                const uint32_t tb = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(QW * qg);
#pragma unroll
                for (int c = 0; c < QW / 32; ++c) {
                    const int ch = qg * (QW / 32) + c;
                    if (c < ncq) {
                        uint32_t v[32];
                        tmem_ld<32>(tb + c * 32, v);
                        tmem_wait();
#pragma unroll
                        for (int g = 0; g < 8; ++g)
                            gm[ch * 8 + g] =
                                max3(__uint_as_float(v[4 * g]), __uint_as_float(v[4 * g + 1]),
                                     fmaxf(__uint_as_float(v[4 * g + 2]), __uint_as_float(v[4 * g + 3])));
                    } else {
#pragma unroll
                        for (int g = 0; g < 8; ++g) gm[ch * 8 + g] = -0x1p120f;
                    }
                }
                if (qg < nq) {  // this accumulator is consumed: the next tile's MMAs may refill it
                    tc_fence_before();
                    mbar_arrive(&dempty[qg]);
                }
            }
            float vm[8];
#pragma unroll
            for (int u = 0; u < 8; ++u)
                vm[u] = max3(max3(gm[8 * u], gm[8 * u + 1], gm[8 * u + 2]), max3(gm[8 * u + 3], gm[8 * u + 4], gm[8 * u + 5]),
                             fmaxf(gm[8 * u + 6], gm[8 * u + 7]));
            const float vmax = max3(max3(vm[0], vm[1], vm[2]), max3(vm[3], vm[4], vm[5]), fmaxf(vm[6], vm[7]));
            float E, Qa;  // from the converter (stage i % BS is recycled only after this tile's reduction)
            asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(E), "=f"(Qa)
                         : "r"(sbase + OFF_EQ + ((uint32_t)(i % BS) * TM + r) * 8) : "memory");
            const float Dhat = fmaxf(Qa - 2.f * vmax, 0.f);
            const float T = (2.f * E + 0x1p-16f * Dhat) * 1.001f;
            // candidate group <=> its maximum >= vmax - T <=> > thr (next float below vmax - T);
            // the sign bits of thr - gm are funnel-shifted into masks (bit 31 - g <-> group g)
            const float thr = next_below(vmax - T);
            uint32_t mk0 = 0, mk1 = 0;
            const uint64_t thr2 = pk2(thr, thr);
#pragma unroll
            for (int g = 0; g < 32; g += 2) {  // packed: two groups per FADD2 (each lane rounds alone)
                float d0, d1, d2, d3;
                upk2(sub2(thr2, pk2(gm[g], gm[g + 1])), d0, d1);
                upk2(sub2(thr2, pk2(gm[32 + g], gm[32 + g + 1])), d2, d3);
                mk0 = __funnelshift_l(__float_as_uint(d0), mk0, 1);
                mk1 = __funnelshift_l(__float_as_uint(d2), mk1, 1);
                mk0 = __funnelshift_l(__float_as_uint(d1), mk0, 1);
                mk1 = __funnelshift_l(__float_as_uint(d3), mk1, 1);
            }
            // exact re-check of the candidate groups in ascending centroid order (strict <)
            float bd = __int_as_float(0x7f800000);
            int bi = 0;
            while (mk0 | mk1) {
                int G;
                if (mk0) { G = __clz(mk0); mk0 &= ~(0x80000000u >> G); }
                else { G = 32 + __clz(mk1); mk1 &= ~(0x80000000u >> (G - 32)); }
                const uint32_t gb = sPC + G * kGrpBytes;
                uint64_t acc0 = 0ull, acc1 = 0ull;  // (4G, 4G+1), (4G+2, 4G+3)
#pragma unroll
                for (int j = 0; j < 16; j += 2) {
                    const float4 c0 = lds_f4(gb + j * 8);
                    const float4 c1 = lds_f4(gb + 128 + j * 8);
                    const uint64_t xa = pk2(xv[j], xv[j]), xb = pk2(xv[j + 1], xv[j + 1]);
                    uint64_t d = add2(xa, pk2(c0.x, c0.y));
                    acc0 = fma2(d, d, acc0);
                    d = add2(xa, pk2(c1.x, c1.y));
                    acc1 = fma2(d, d, acc1);
                    d = add2(xb, pk2(c0.z, c0.w));
                    acc0 = fma2(d, d, acc0);
                    d = add2(xb, pk2(c1.z, c1.w));
                    acc1 = fma2(d, d, acc1);
                }
                float dd[4];
                upk2(acc0, dd[0], dd[1]);
                upk2(acc1, dd[2], dd[3]);
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    const int c = 4 * G + e;
                    if (c < kc && dd[e] < bd) { bd = dd[e]; bi = c; }
                }
            }
            if (valid) member[p] = bi;
            // the point's one-hot byte (cluster row bi, point column r); the byte this thread set
            // in this stage OS tiles ago is cleared first
            const int o = (int)(i % OS);
            mbar_wait(&oempty[o], (uint32_t)((i / OS) & 1) ^ 1u);
            int32_t& pd = (o == 0) ? pend[0] : pend[1];
            if (pd >= 0) sts_u8(sOH + o * kOHBytes + (uint32_t)pd, 0u);
            if (valid) {
                const uint32_t off = (uint32_t)(bi >> 7) * 16384u + sw_off((uint32_t)(bi & 127), (uint32_t)r);
                sts_u8(sOH + o * kOHBytes + off, 1u);
                pd = (int32_t)off;
            } else {
                pd = -1;
            }
            fence_async_smem();
            mbar_arrive(&ofull[o]);
        }
        // reduction accumulators: lane = cluster (h*128 + r), columns 4j+b = byte sums, 64 = count
        mbar_wait(sdone, 0);
        tc_fence_after();
        for (int h = 0; h < nh; ++h) {
            uint32_t v0[32], v1[32], v2[16];
            const uint32_t tb = tmem + ((uint32_t)(q * 32) << 16) + kColSum + 80u * h;
            tmem_ld<32>(tb, v0);
            tmem_ld<32>(tb + 32, v1);
            tmem_ld<16>(tb + 64, v2);
            tmem_wait();
            const int c = 128 * h + r;
            const uint64_t cnt = v2[0];
            if (c < kc && cnt) {
#pragma unroll
                for (int j = 0; j < 16; ++j) {
                    const uint32_t* w = j < 8 ? &v0[4 * j] : &v1[4 * (j - 8)];
                    const uint64_t su = (uint64_t)w[0] + ((uint64_t)w[1] << 8) + ((uint64_t)w[2] << 16) +
                                        ((uint64_t)w[3] << 24);
                    const int64_t sv = (int64_t)(su - (cnt << 31));  // remove the 2^31 bias
                    if (sv) atomicAdd(reinterpret_cast<unsigned long long*>(sums) + c * 16 + j, (unsigned long long)sv);
                }
                atomicAdd(reinterpret_cast<unsigned long long*>(counts) + c, (unsigned long long)cnt);
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

}  // namespace

int kmeans_tc_supported(const float* x, int d, int kc) {
    return d == 16 && kc >= 1 && kc <= KMAX && (reinterpret_cast<uintptr_t>(x) % 16) == 0;
}

cudaError_t kmeans_assign_tc(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                             int64_t p0, int64_t p1, int kc, int shift, int* err_flag, cudaStream_t s, int sms) {
    if (p1 <= p0) return cudaSuccess;
    if (p1 - p0 > (int64_t)INT32_MAX - TM) return cudaErrorNotSupported;  // TMA row coordinates are int32
    const int npad = ((kc + 31) / 32) * 32;
    // accumulator group width (ACCMG_KMEANS_TC_QW: 32, 64 or 128 centroid columns; same-box A/B in
    // profiles/r01/kmeans_tc.log: 128 = 22.9 ms, 64 = 29.4, 32 = 42.4 — more, narrower MMAs lose)
    static int qw = -1;
    if (qw < 0) {
        const char* v = getenv("ACCMG_KMEANS_TC_QW");
        qw = v ? atoi(v) : 128;
    }
    auto kern = qw == 64 ? assign_tc<64> : qw == 32 ? assign_tc<32> : assign_tc<128>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemTC);
    if (e != cudaSuccess) return e;
    const int64_t ntiles = (p1 - p0 + TM - 1) / TM;
    // s32 reduction accumulators: byte sums <= 255 per point, so at most 2^23 points (65536 tiles)
    // per CTA; more CTAs than SMs run in waves
    int64_t blocks = ntiles < sms ? ntiles : sms;
    const int64_t need = (ntiles + 65535) / 65536;
    if (blocks < need) blocks = need;
    // point tiles by TMA: [rows][16] fp32 from p0, 128-row boxes, 64-byte swizzle (the per-row
    // float4 reads of the converter and epilogue threads hit 8 distinct bank groups)
    auto fn = tma_encode_fn();
    if (!fn) return cudaErrorNotSupported;
    CUtensorMap xmap;
    cuuint64_t dims[2] = {16, (cuuint64_t)(p1 - p0)};
    cuuint64_t strides[1] = {64};
    cuuint32_t box[2] = {16, TM};
    cuuint32_t es[2] = {1, 1};
    if (fn(&xmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(x) + p0 * 16, dims, strides, box, es,
           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return cudaErrorNotSupported;
    kern<<<(unsigned)blocks, kThreadsTC, kSmemTC, s>>>(xmap, cen, member, sums, counts, p0, p1, kc, npad, shift,
                                                            err_flag);
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
