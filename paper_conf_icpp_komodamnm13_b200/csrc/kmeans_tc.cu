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
//     accumulator (a ring of three 128-column TMEM slots), so the next tile's MMAs overlap the
//     epilogue's reads of this one;
//   * reductiontoarray: sums[c][(j, b)] = sum_p onehot[c][p] * byte_b(x[p][j] * 2^shift + 2^31) and
//     counts[c] = sum_p onehot[c][p] * 1 — tcgen05.mma.kind::i8 (u8 x u8 -> s32, exact) with
//     A = the one-hot assignment matrix [128 clusters][128 points] and B = the points' fixed-point
//     byte planes [64 rows (j, b)][128 points] (MN-major: a point's 64 bytes are its 16 words); the
//     s32 accumulators stay in TMEM across all the CTA's tiles and are read once at the end; the
//     counts are shared-memory integer atomics (no per-point global atomics).
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
// Warp roles (one CTA per SM, persistent over 128-point tiles; 16 warps):
//   w0 producer: TMA load (64-byte swizzle) of the tile's fp32 rows (8 KiB) into an mbarrier ring;
//   w15 / w1 distance-MMA issuers (centroid halves 0 / 1), w14 reduction-MMA issuer (one tile behind);
//   w2-5 converters (one point per thread): bf16 pieces of x into the distance A operand, the
//        fixed-point words into the reduction B operand, the 2^-shift grid check, the point's
//        bound terms E and Q(1 + 2^-17) + 2E for the epilogue;
//   w6-13 epilogue, two sets of four (one per centroid half; warp % 4 = TMEM lane quarter, one point
//        per thread): maxima over the orthogonal column groupings, one exchange of the halves'
//        maxima and verdicts, the exact re-check only when the candidate is not proved unique,
//        member[p], the count atomic and the point's one-hot byte.
// DESIGN.md §6 has the measurements behind this layout.
#include <cuda_bf16.h>

#include <cstdio>
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
#ifndef KM_DEBUG_HANG
using dev::mbar_wait;
#endif
using dev::smem_u32;

constexpr int TM = 128;                 // points per tile (distance MMA M, reduction MMA K)
constexpr int KMAX = 256;               // centroids
constexpr int XS = 4;                   // fp32 point-tile stages
constexpr int AS = 2;                   // distance A operand stages in TMEM (freed by the distance MMAs)
constexpr int BS = 4;                   // reduction B operand stages (freed by the reduction MMAs)
constexpr int OS = 2;                   // one-hot stages
constexpr int kRows = 32;               // reduction B rows: 16 dims x 2 bytes (counts: shared atomics)
constexpr int kXBytes = TM * 64;        // 8 KiB
constexpr int kABBytes = kRows * TM;    // 4 KiB: MN-major, point p's 32 bytes (16 dims x 2 bytes) at row p
constexpr int kOHBytes = KMAX * 128;    // 32 KiB (two 128-cluster halves)
constexpr int QW = 128;                 // centroid columns per distance accumulator (one MMA N)
constexpr int NDB = 3;                  // distance accumulators: a ring of three 128-column halves
// warps (sub-partition = warp % 4): 0 producer, 2-5 converters, 6-13 epilogue (two sets of four:
// warp % 4 is the TMEM lane quarter), 15 / 1 distance-MMA issuers (centroid halves 0 / 1), 14
// reduction-MMA issuer. A tcgen05.mma holds back its issuing sub-partition's other warps while it
// runs (scripts/km_trace.cu: the epilogue warp beside the MMA issuer lagged ~1000 cycles per tile),
// so the three MMA streams sit on the three sub-partitions the producer does not use
constexpr int kThreadsTC = 512;
constexpr int kRedWarp = 14;
constexpr int kTmemCols = 512;
constexpr uint32_t kColSum = NDB * QW;  // reduction accumulators: cluster half h at 384 + 32 h

constexpr int OFF_AB = 0;
constexpr int OFF_BD = OFF_AB + BS * kABBytes;
constexpr int OFF_OH = OFF_BD + KMAX * 128;
constexpr int OFF_X = OFF_OH + OS * kOHBytes;
// re-check copy of the centroids, negated, for packed pairs: group G = centroids 4G..4G+3 at
// G * kGrpBytes (16 B of padding per group spreads the lanes' groups over the banks), pair P of
// the group at +128 P, dims (j, j+1) of both centroids of the pair at +8 j: one LDS.128
constexpr int kGrpBytes = 272;
constexpr int OFF_PC = OFF_X + XS * kXBytes;
constexpr int OFF_BAR = OFF_PC + (KMAX / 4) * kGrpBytes;
constexpr int kNumBars = 2 * XS + 2 * AS + BS + 2 * NDB + 2 * OS + 3;
constexpr int OFF_MISC = OFF_BAR + kNumBars * 8;    // tmem slot, Cinf bits, C2 bits
constexpr int OFF_EQ = OFF_MISC + 16;               // float2 [BS][TM]: the point's E and Q (1 + 2^-17) + 2E
constexpr int OFF_CNT = OFF_EQ + BS * TM * 8;       // int32 [KMAX]: the CTA's cluster counts
constexpr int kSmemTC = OFF_CNT + KMAX * 4 + 1024;  // + alignment slack
static_assert(OFF_AB % 1024 == 0 && OFF_BD % 1024 == 0 && OFF_OH % 1024 == 0 && OFF_X % 1024 == 0, "align");
// distance A operand in TMEM (lane = point): the constant slice [1 1 1 0 ...] (8 columns of bf16
// pairs) and AS stages of [x0 (8 columns) | x1 (8 columns)]
constexpr uint32_t kColA1 = kColSum + 2 * kRows;
constexpr uint32_t kColA = kColA1 + 8;
static_assert(kColA + AS * 16 <= kTmemCols, "tmem");
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
// warp-collective forms: every lane executes them with the same operands, one elected lane issues
// A from tensor memory (K-major, lane = row): [d], [a], b-desc
__device__ __forceinline__ void mma_f16_ts_elect(uint32_t d, uint32_t a_tmem, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\tsetp.ne.b32 p, %4, 0;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
        "r"(a_tmem), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void mma_i8_elect(uint32_t d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\tsetp.ne.b32 p, %4, 0;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void tc_commit_elect(uint64_t* bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
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
// MN-major operand, 32-byte swizzle, N = 32 one-byte elements: K row p (32 B) at 32 p, 8-row atoms
// 256 B apart (SBO); one atom along N, so the leading-dimension offset is never stepped
__device__ __forceinline__ uint64_t sdesc_mn_sw32(uint32_t saddr) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)(kABBytes >> 4) << 16;
    d |= (uint64_t)(256 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)6 << 61;
    return d;
}
// byte offset of element k (byte k) of row m in a 128-byte-swizzled K-major operand
__device__ __forceinline__ uint32_t sw_off(uint32_t m, uint32_t kbyte) {
    return m * 128u + ((((kbyte >> 4) ^ (m & 7u)) << 4) | (kbyte & 15u));
}
// wait with a suspend-time hint: a warp that waits for a free stage sleeps instead of spinning on
// issue slots the converter / epilogue warps of its SM sub-partition need
#ifdef KM_DEBUG_HANG  // waits that report themselves and trap after ~2^26 polls (debug builds only)
__device__ __forceinline__ void mbar_wait_dbg(uint64_t* bar, uint32_t parity, int line) {
    for (uint32_t it = 0;; ++it) {
        uint32_t ok;
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
        if (ok) return;
        if (it == (1u << 24)) {
            printf("hang: block %d warp %d lane %d line %d bar %u parity %u\n", blockIdx.x, threadIdx.x / 32,
                   threadIdx.x % 32, line, smem_u32(bar) & 0xFFFF, parity);
            __trap();
        }
    }
}
#define mbar_wait_sleep(b, p) mbar_wait_dbg(b, p, __LINE__)
#define mbar_wait(b, p) mbar_wait_dbg(b, p, __LINE__)
#else
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAITS_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
        "@!p bra WAITS_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity), "r"(20000u)
        : "memory");
}
#endif
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
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
        "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
        : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&r)[8]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(r[0]),
                 "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
                 : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

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

#ifdef KM_PROGRESS  // per-warp progress in mapped host memory (scripts/km_hang.cu); debug builds only
__device__ unsigned* g_prog;
#define KPR(EV, T)                                                                                     \
    do {                                                                                             \
        if ((threadIdx.x & 31) == 0 && blockIdx.x < 4096)                                            \
            *(volatile unsigned*)&g_prog[blockIdx.x * 16 + (threadIdx.x >> 5)] = ((EV) << 24) | (T);  \
    } while (0)
#else
#define KPR(EV, T)
#endif
#ifndef KTR_EPI
#define KTR_EPI 6  // epilogue warp whose events the trace records (its half-1 partner: KTR_EPI + 4)
#endif
#ifdef KM_TRACE  // per-role timeline of CTA 0 (scripts/km_trace.cu); compiled out of the product
__device__ unsigned long long g_km_trace[64][32];
#define KTR(W, EV)                                                                                   \
    do {                                                                                             \
        if (blockIdx.x == 0 && warp == (W) && lane == 0 && i >= 200 && i < 264)                      \
            g_km_trace[i - 200][EV] = clock64();                                                     \
    } while (0)
#else
#define KTR(W, EV)
#endif

constexpr int kProdWarp = 0, kMmaWarp = 15, kMmaWarp1 = 1;

// exact mode: v added exactly into two of the nine 32-bit-aligned int64 windows of its sum
// (weight of window w: 2^(32 w - 149)); the same representation as kmeans.cu's exact kernels
// (the converter has rejected non-finite points)
__device__ __forceinline__ void superacc_add_tc(unsigned long long* acc, float v) {
    const uint32_t b = __float_as_uint(v);
    const uint32_t ex = (b >> 23) & 255u;
    uint32_t m = b & 0x7FFFFFu;
    if (ex) m |= 0x800000u;
    if (!m || ex == 255u) return;
    const int o = ex ? (int)ex - 1 : 0;
    const uint64_t t = (uint64_t)m << (o & 31);
    unsigned long long lo = t & 0xFFFFFFFFull, hi = t >> 32;
    if (b >> 31) {
        lo = 0ull - lo;
        hi = 0ull - hi;
    }
    if (lo) atomicAdd(acc + (o >> 5), lo);
    if (hi) atomicAdd(acc + (o >> 5) + 1, hi);
}

__device__ __forceinline__ void named_bar(uint32_t id, uint32_t n) {
    // non-aligned form: a warp may arrive diverged (after data-dependent re-check loops)
    __syncwarp();
    asm volatile("barrier.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}

// Two epilogue warps per TMEM lane quarter, one per 128-centroid half: a single warp's tcgen05.ld
// + wait::ld sustains ~32 B/cycle (scripts/tmem_bw.cu), so one warp would need ~1000 cycles per
// tile for the 128 KiB of distances. The distance accumulators form a ring of three 128-column
// buffers (half h of tile i in buffer (nq i + h) mod 3), so the MMAs of the next tile's first half
// run while the epilogue still reads this tile's two halves.
// EXACT (shift = ACCMG_KMEANS_EXACT, reading KM-X): any finite points. The assignment is the same
// filter + exact re-check; a point with |x| > 2^60 (or centroids beyond 2^60, where x.c could
// overflow the fp32 accumulation) skips the filter and re-checks every centroid. The sums go to
// nine 32-bit-aligned int64 windows per (cluster, dim) through the epilogue's global-atomic path
// (every point takes it: no fixed-point words for the reduction MMA).
template <bool EXACT>
__global__ void __launch_bounds__(kThreadsTC, 1)
assign_tc(const __grid_constant__ CUtensorMap xmap, const float* __restrict__ xg, const float* __restrict__ cen,
          int32_t* __restrict__ member,
          int64_t* __restrict__ sums, int64_t* __restrict__ counts, int64_t p0, int64_t p1, int kc, int npad,
          int shift, int* err) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    // aligned base inside the shared window (address arithmetic on smem_raw keeps the state space)
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t pad = ((raw + 1023u) & ~1023u) - raw;
    unsigned char* smem = smem_raw + pad;
    const uint32_t sbase = raw + pad;
    const uint32_t sAB = sbase + OFF_AB, sBD = sbase + OFF_BD, sOH = sbase + OFF_OH;
    const uint32_t sX = sbase + OFF_X, sPC = sbase + OFF_PC;
    uint64_t* xfull = reinterpret_cast<uint64_t*>(smem + OFF_BAR);
    uint64_t* xempty = xfull + XS;
    uint64_t* afull = xempty + XS;
    uint64_t* aempty = afull + AS;
    uint64_t* bempty = aempty + AS;
    uint64_t* dfull = bempty + BS;
    uint64_t* dempty = dfull + NDB;
    uint64_t* ofull = dempty + NDB;
    uint64_t* oempty = ofull + OS;
    uint64_t* sdone = oempty + OS;
    uint64_t* h1go = sdone + 1;  // phase i: the half-1 MMAs of tile i are issued
    uint64_t* h0go = h1go + 1;   // phase i: the half-0 MMAs of tile i are issued
    uint32_t* misc = reinterpret_cast<uint32_t*>(smem + OFF_MISC);  // [0] tmem, [1] Cinf bits, [2] C2 bits

    constexpr int kThreads = kThreadsTC;
    // the warp index through a shuffle: the compiler then treats the role branches as warp-uniform
    // (descriptors and loop state of the MMA issuers stay in uniform registers; 8.5 % faster)
    const int tid = threadIdx.x, warp = __shfl_sync(0xffffffffu, tid >> 5, 0), lane = tid & 31;
    const int64_t ntiles = (p1 - p0 + TM - 1) / TM;
    const int64_t nt = blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
    const uint32_t nt32 = (uint32_t)nt;
    const int nh = (npad + 127) / 128;  // 128-centroid halves (reduction)
    const int nq = nh;                  // distance accumulator halves per tile

    // ---- setup: constant operand parts, centroids, bounds, barriers, TMEM
    if (tid == 0) { misc[1] = 0u; misc[2] = 0u; }
    for (int i = tid; i < npad * 16; i += kThreads) {
        const int c = i >> 4, j = i & 15;
        const float v = c < kc ? -cen[i] : 0.f;
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sPC + (c >> 2) * kGrpBytes + ((c >> 1) & 1) * 128 + j * 8 +
                                                    (c & 1) * 4),
                     "f"(v)
                     : "memory");
    }
    for (uint32_t i = tid; i < OS * kOHBytes / 16; i += kThreads) sts_v4(sOH + i * 16, make_uint4(0, 0, 0, 0));
    for (int i = tid; i < KMAX; i += kThreads) reinterpret_cast<int*>(smem + OFF_CNT)[i] = 0;
    if (tid == 0) {
        for (int s = 0; s < XS; ++s) { mbar_init(&xfull[s], 1); mbar_init(&xempty[s], 128); }  // the converters
        for (int a = 0; a < AS; ++a) { mbar_init(&afull[a], 128); mbar_init(&aempty[a], nq); }  // nq issuers
        for (int b = 0; b < BS; ++b) mbar_init(&bempty[b], 1);
        for (int b = 0; b < NDB; ++b) { mbar_init(&dfull[b], 1); mbar_init(&dempty[b], 128); }
        for (int o = 0; o < OS; ++o) { mbar_init(&ofull[o], 128); mbar_init(&oempty[o], 1); }
        mbar_init(sdone, 1);
        mbar_init(h1go, 1);
        mbar_init(h0go, 1);
        dev::mbar_fence_init();
    }
    KPR(1, 0);
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(misc)),
                     "r"(kTmemCols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    __syncthreads();
    for (int n = tid; n < npad; n += kThreads) {  // distance B rows [c0 | c1 | c0 | h0 h1 h2 0 ...]
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
    KPR(2, 0);
    __syncthreads();
    tc_fence_after();
    KPR(3, 0);
    const uint32_t tmem = misc[0];

    // reductiontoarray MMAs of tile j (u8 one-hot x byte planes -> s32, B MN-major), issued by one
    // warp after the epilogue has filled the tile's one-hot stage
    auto issue_reduction = [&](uint32_t j) {
        const uint32_t idesc_sum = (2u << 4) | (1u << 16) | ((uint32_t)(kRows >> 3) << 17) | ((uint32_t)(TM >> 4) << 24);
        const uint64_t dAB = sdesc_mn_sw32(sAB), dOH = sdesc_sw128(sOH);
        const int o = (int)(j % OS);
        mbar_wait_sleep(&ofull[o], (uint32_t)((j / OS) & 1));
        KPR(8, j);
        tc_fence_after();
        const uint64_t b = dAB + (uint64_t)(((j % BS) * kABBytes) >> 4);
        const uint64_t oh = dOH + (uint64_t)((o * kOHBytes) >> 4);
        for (int h = 0; h < nh; ++h)
#pragma unroll
            for (int k = 0; k < 4; ++k)
                mma_i8_elect(tmem + kColSum + (uint32_t)(kRows * h), oh + (uint64_t)((h * 16384 + k * 32) >> 4),
                             b + (uint64_t)((k * 32 * kRows) >> 4), idesc_sum, (j | k) ? 1u : 0u);
        tc_commit_elect(&oempty[o]);
        tc_commit_elect(&bempty[j % BS]);
        KPR(9, j);
    };
    if (warp == kProdWarp) {
        // ---- producer
        if (lane == 0) {
            for (uint32_t i = 0; i < nt32; ++i) {
                const uint32_t t = blockIdx.x + i * gridDim.x;
                const int s = (int)(i % XS);
                mbar_wait_sleep(&xempty[s], (uint32_t)((i / XS) & 1) ^ 1u);
                KTR(kProdWarp, 25);
                KPR(4, i);
                mbar_expect_tx(&xfull[s], kXBytes);  // rows past the end are zero-filled
                dev::tma_load_2d(&xmap, &xfull[s], smem + OFF_X + s * kXBytes, 0, (int)(t * TM));
            }
        }
    } else if (warp == kMmaWarp || warp == kMmaWarp1) {
        // ---- distance-MMA issuers, one per 128-centroid half (tcgen05.mma occupies the issuing
        // sub-partition while it runs, so the three MMA streams sit on three sub-partitions). The
        // whole warp runs the loop and one elected lane issues each tcgen05 instruction;
        // descriptors are the stage bases plus the 16-byte-unit offsets of the slices
        const int h = warp == kMmaWarp ? 0 : 1;
        const uint64_t dBD = sdesc_sw128(sBD);
        const int wq = (npad - QW * h) < QW ? (npad - QW * h) : QW;
        const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(wq >> 3) << 17) |
                               ((uint32_t)(TM >> 4) << 24);
        const uint64_t bd = dBD + (uint64_t)((h * QW * 128) >> 4);
        for (uint32_t i = 0; i < nt32 && h < nq; ++i) {
            const int a = (int)(i % AS);
            mbar_wait_sleep(&afull[a], (uint32_t)((i / AS) & 1));
            KTR(kMmaWarp, 4);
            KPR(5, i);
            const uint32_t at = tmem + kColA + 16u * (uint32_t)a;  // this tile's [x0 | x1] in TMEM
            const uint32_t u = (uint32_t)nq * i + (uint32_t)h, db = u % NDB;  // ring slot and its use count
            // the tensor pipe takes MMAs in issue order and the epilogue reads the halves in ring
            // order: the two streams alternate strictly (half 0 of tile i after half 1 of tile i-1,
            // half 1 of tile i after half 0 of tile i)
            if (h == 0 && nq == 2 && i > 0) mbar_wait_sleep(h1go, (i - 1) & 1u);
            if (h == 1) mbar_wait_sleep(h0go, i & 1u);
            mbar_wait_sleep(&dempty[db], ((u / NDB) & 1u) ^ 1u);
            KTR(kMmaWarp, 5);
            KTR(kMmaWarp1, 6);
            KPR(6, i);
            tc_fence_after();
#pragma unroll
            for (int k = 0; k < 4; ++k)
                // A slices x0, x0, x1, 1 (from TMEM; x0 read twice) against B slices c0, c1, c0, h
                mma_f16_ts_elect(tmem + QW * db, k == 3 ? tmem + kColA1 : at + (k == 2 ? 8u : 0u),
                                 bd + (uint64_t)((k * 32) >> 4), idesc, k ? 1u : 0u);
            tc_commit_elect(&dfull[db]);
            tc_commit_elect(&aempty[a]);
            __syncwarp();
            if (lane == 0 && nq == 2) mbar_arrive(h == 1 ? h1go : h0go);
            KPR(7, i);
            KTR(kMmaWarp, 13);
            KTR(kMmaWarp1, 14);
        }
    } else if (warp == kRedWarp) {
        // (issuing the reductions from the last distance stream, right after its group, measured
        // 4 % slower: scripts/r2_kab.sh)
        for (uint32_t j = 0; j < nt32; ++j) issue_reduction(j);
        tc_commit_elect(sdone);
        KPR(10, 0);
    } else if (warp >= 2 && warp < 6) {
        // ---- converters: point row r = TMEM lane of the warp's lane quarter (warp % 4)
        const int r = 32 * (warp & 3) + lane;
        const uint32_t tqc = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
        {  // the constant A slice [1 1 1 0 ... 0] (bf16 ones: the -|c|^2/2 pieces h0 + h1 + h2)
            const uint32_t ones[8] = {0x3F803F80u, 0x00003F80u, 0u, 0u, 0u, 0u, 0u, 0u};
            tmem_st8(tqc + kColA1, ones);
            tmem_wait_st();
        }
        const float scale = EXACT ? 1.f : (float)(1 << shift);
        const float Cinf = __uint_as_float(misc[1]);
        const float C2 = __uint_as_float(misc[2]);
        int bad = 0;
        for (uint32_t i = 0; i < nt32; ++i) {
            const int s = (int)(i % XS), a = (int)(i % AS);
            mbar_wait_sleep(&xfull[s], (uint32_t)((i / XS) & 1));
            KTR(2, 0);
            KPR(11, i);
            float xv[16];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const float4 v = lds_f4(sX + s * kXBytes + r * 64 + ((j ^ ((r >> 1) & 3)) << 4));
                xv[4 * j] = v.x; xv[4 * j + 1] = v.y; xv[4 * j + 2] = v.z; xv[4 * j + 3] = v.w;
            }
            mbar_wait_sleep(&aempty[a], (uint32_t)((i / AS) & 1) ^ 1u);
            tc_fence_after();
            KTR(2, 1);
            KPR(12, i);
            const int bs = (int)(i % BS);
            mbar_wait_sleep(&bempty[bs], (uint32_t)((i / BS) & 1) ^ 1u);
            KTR(2, 2);
            KPR(13, i);
            uint4 h0, l0, h1, l1;
            split8(xv, h0, l0);
            split8(xv + 8, h1, l1);
            {  // [x0 | x1] of the point into its TMEM lane (the MMA reads x0 twice)
                const uint32_t w[16] = {h0.x, h0.y, h0.z, h0.w, h1.x, h1.y, h1.z, h1.w,
                                        l0.x, l0.y, l0.z, l0.w, l1.x, l1.y, l1.z, l1.w};
                tmem_st16(tqc + kColA + 16u * (uint32_t)a, w);
            }
            // the stage is released only after instructions that consume the loaded values (the
            // arrive alone does not wait for the shared-memory loads to return their data, and the
            // producer refills the stage as soon as all converters have arrived)
            mbar_arrive(&xempty[s]);
            // fixed point v = x * 2^shift, as 16-bit words biased to unsigned: u = v + 2^15 when every
            // |v_j| < 2^15 (the point "fits"); otherwise u = 2^15 (v taken as 0 here) and the point is
            // flagged for the exact int64 path in the epilogue. The B operand is MN-major: the point's
            // 32 bytes in order (j, b) are its 16 halfwords, little-endian, so two 16-byte stores write
            // the row (32-byte swizzle: chunk c of row r at c ^ ((r >> 2) & 1)).
            // Grid check without branches: v must equal rint(v) (every float of magnitude >= 2^23 is
            // an integer) and |v| < 2^31; the largest |v - rint(v)| and |v| of the point are tested once
            float fr = 0.f, vm = 0.f;
            int iv[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const float v = xv[j] * scale;  // exact: power-of-two scaling
                const float rv = rintf(v);
                fr = fmaxf(fr, fabsf(v - rv));  // exact difference (Sterbenz)
                vm = fmaxf(vm, fabsf(v));
                iv[j] = __float2int_rn(rv);
            }
            const bool fits = !EXACT && vm < 32768.0f;
            {
                uint32_t hw[8];
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    hw[j] = fits ? __byte_perm((uint32_t)iv[2 * j] ^ 0x8000u, (uint32_t)iv[2 * j + 1] ^ 0x8000u, 0x5410)
                                 : 0x80008000u;
                const uint32_t row = sAB + bs * kABBytes + (uint32_t)r * 32u, sw = ((uint32_t)r >> 2) & 1u;
                sts_v4(row + ((0u ^ sw) << 4), make_uint4(hw[0], hw[1], hw[2], hw[3]));
                sts_v4(row + ((1u ^ sw) << 4), make_uint4(hw[4], hw[5], hw[6], hw[7]));
            }
            if constexpr (EXACT) {
                bool nf = false;
#pragma unroll
                for (int j = 0; j < 16; ++j) nf |= !(fabsf(xv[j]) <= 3.40282347e38f);  // inf or NaN
                bad |= nf;
            } else {
                bad |= (fr != 0.f) | !(vm < 2147483648.0f);
            }
            {  // the filter bound's per-point terms, for the epilogue (header: E, Dhat)
                float L1 = 0.f, Q = 0.f;
#pragma unroll
                for (int j = 0; j < 16; ++j) { L1 += fabsf(xv[j]); Q = fmaf(xv[j], xv[j], Q); }
                const float E = (0x1p-11f * (L1 * Cinf + C2)) * 1.001f + 0x1p-100f;
                const float Qa = Q * (1.f + 0x1p-17f) + 2.f * E;
                // (the sign of E carries the point's "does not fit" flag; E > 0)
                // exact mode: E = -inf marks a point whose distances the filter cannot bound
                const bool unsafe = EXACT && !(vm <= 0x1p60f && Cinf <= 0x1p60f);
                asm volatile("st.shared.v2.f32 [%0], {%1, %2};" ::"r"(sbase + OFF_EQ + (bs * TM + r) * 8),
                             "f"(unsafe ? -__int_as_float(0x7f800000) : (fits ? E : -E)), "f"(Qa)
                             : "memory");
            }
            fence_async_smem();  // the B operand (shared memory) for the reduction MMAs
            tmem_wait_st();      // the A operand (TMEM) for the distance MMAs
            tc_fence_before();
            mbar_arrive(&afull[a]);
            KTR(2, 3);
            KPR(14, i);
        }
        if (bad) atomicOr(err, 1);
    } else if (warp >= 6 && warp < 14) {
        // ---- epilogue: two sets of four warps take alternate tiles (set = tile parity), so each
        // set has two tile periods for its tile and the sets never wait for each other. Point row
        // r = TMEM lane (warp % 4 = lane quarter); the thread reads all k columns of its point
        // (one 128-column ring slot per half, freed as soon as it is read) and keeps the maxima of
        // two orthogonal column groupings of the 16 x 16 grid l = 16 b + a: b-groups (16
        // consecutive columns) and a-groups (columns with the same l mod 16). (a, b) names one
        // column, so when exactly one a-group and one b-group reach the threshold the candidate
        // set is that single column: the argmin is proved without any re-check (the common case
        // for separated clusters). Otherwise every 4-column group of the product set (candidate
        // b-groups x quarters holding candidate a-groups) is re-checked with the exact fmaf chain.
        const int q = warp & 3;
        const int r = q * 32 + lane;
        const int half = (warp - 6) >> 2;  // the set (also its share of the final readout)
        const int o = half;                // one-hot stage of the set's tiles (tile parity)
        int* s_cnt = reinterpret_cast<int*>(smem + OFF_CNT);  // the CTA's cluster counts
        int32_t pend = -1;                 // the one-hot byte this thread set in its stage
        const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16);
        for (uint32_t i = (uint32_t)half; i < nt32; i += 2) {
            const uint32_t t = blockIdx.x + i * gridDim.x;
            const uint32_t pr = t * TM + (uint32_t)r;  // row within the partition (< 2^31)
            const int64_t p = p0 + pr;
            const bool valid = pr < (uint32_t)(p1 - p0);
            KTR(KTR_EPI, 9);
            KTR(KTR_EPI + 4, 21);
            KPR(15, i);
            float am[16], bm[16];  // set by the first chunk (h = 0 always has one); -2^120 = no column
            // software-pipelined read: 32-column chunks g = 4 h + c, chunk g + 1 in flight while chunk
            // g is reduced (tcgen05.wait::ld waits for all of the thread's loads, so one ahead)
            const int ncq0 = (npad < QW ? npad : QW) / 32;
            const int ncq1 = nq == 2 ? (npad - QW) / 32 : 0;
            const uint32_t u0 = (uint32_t)nq * i, db0 = u0 % NDB, db1 = (u0 + 1) % NDB;
            mbar_wait(&dfull[db0], (u0 / NDB) & 1u);
            tc_fence_after();
            KTR(KTR_EPI, 11);
            KTR(KTR_EPI + 4, 22);
            KPR(16, i);
            uint32_t va[32], vb[32];
            tmem_ld<32>(tq + QW * db0, va);
            tmem_wait();
#pragma unroll
            for (int g = 0; g < 8; ++g) {
                const int h = g >> 2, c = g & 3;
                uint32_t(&cur)[32] = (g & 1) ? vb : va;
                uint32_t(&nxt)[32] = (g & 1) ? va : vb;
                const bool have = h == 0 ? c < ncq0 : c < ncq1;
                const int gn = g + 1, hn = gn >> 2, cn = gn & 3;
                const bool have_n = gn < 8 && (hn == 0 ? cn < ncq0 : cn < ncq1);
                if (gn == 4 && have_n) {  // half 0 fully read: hand its slot back, wait for half 1
                    tc_fence_before();
                    mbar_arrive(&dempty[db0]);
                    const uint32_t u1 = u0 + 1;
                    mbar_wait(&dfull[db1], (u1 / NDB) & 1u);
                    tc_fence_after();
                }
                if (have_n) tmem_ld<32>(tq + QW * (hn ? db1 : db0) + cn * 32, nxt);
                if (have) {
#define VF(k) __uint_as_float(cur[k])
                    bm[2 * g] = max3(max3(max3(VF(0), VF(1), VF(2)), max3(VF(3), VF(4), VF(5)), max3(VF(6), VF(7), VF(8))),
                                     max3(VF(9), VF(10), VF(11)), max3(VF(12), VF(13), fmaxf(VF(14), VF(15))));
                    bm[2 * g + 1] = max3(max3(max3(VF(16), VF(17), VF(18)), max3(VF(19), VF(20), VF(21)),
                                              max3(VF(22), VF(23), VF(24))),
                                         max3(VF(25), VF(26), VF(27)), max3(VF(28), VF(29), fmaxf(VF(30), VF(31))));
                    if (g == 0) {
#pragma unroll
                        for (int a = 0; a < 16; ++a) am[a] = fmaxf(VF(a), VF(16 + a));
                    } else {
#pragma unroll
                        for (int a = 0; a < 16; ++a) am[a] = max3(am[a], VF(a), VF(16 + a));
                    }
#undef VF
                } else {
                    bm[2 * g] = bm[2 * g + 1] = -0x1p120f;
                }
                if (have_n) tmem_wait();
            }
            // every load has completed: the last half's slot goes back to the MMA
            tc_fence_before();
            mbar_arrive(&dempty[nq == 2 ? db1 : db0]);
            KTR(KTR_EPI, 12);
            KTR(KTR_EPI + 4, 23);
            const float vmax = max3(max3(max3(bm[0], bm[1], bm[2]), max3(bm[3], bm[4], bm[5]), max3(bm[6], bm[7], bm[8])),
                                    max3(bm[9], bm[10], bm[11]), max3(bm[12], bm[13], fmaxf(bm[14], bm[15])));
            float E, Qa;  // from the converter (stage i % BS is recycled only after this tile's reduction)
            asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(E), "=f"(Qa)
                         : "r"(sbase + OFF_EQ + ((uint32_t)(i % BS) * TM + r) * 8) : "memory");
            // candidate <=> value >= vmax - T <=> > thr (the next float below)
            const float Dhat = fmaxf(Qa - 2.f * vmax, 0.f);
            const float T = (2.f * fabsf(E) + 0x1p-16f * Dhat) * 1.001f;
            const float thr = next_below(vmax - T);
            // sign bits of thr - max (packed FSUB2, each lane rounds alone) funnel-shifted into the
            // masks: bit 15 - a of mA, bit 15 - b of mB; two independent chains each
            const uint64_t thr2 = pk2(thr, thr);
            uint32_t mA0 = 0, mA1 = 0, mB0 = 0, mB1 = 0;
#pragma unroll
            for (int a = 0; a < 8; a += 2) {
                float d0, d1, d2, d3;
                upk2(sub2(thr2, pk2(am[a], am[a + 1])), d0, d1);
                upk2(sub2(thr2, pk2(am[8 + a], am[9 + a])), d2, d3);
                mA0 = __funnelshift_l(__float_as_uint(d0), mA0, 1);
                mA1 = __funnelshift_l(__float_as_uint(d2), mA1, 1);
                mA0 = __funnelshift_l(__float_as_uint(d1), mA0, 1);
                mA1 = __funnelshift_l(__float_as_uint(d3), mA1, 1);
                upk2(sub2(thr2, pk2(bm[a], bm[a + 1])), d0, d1);
                upk2(sub2(thr2, pk2(bm[8 + a], bm[9 + a])), d2, d3);
                mB0 = __funnelshift_l(__float_as_uint(d0), mB0, 1);
                mB1 = __funnelshift_l(__float_as_uint(d2), mB1, 1);
                mB0 = __funnelshift_l(__float_as_uint(d1), mB0, 1);
                mB1 = __funnelshift_l(__float_as_uint(d3), mB1, 1);
            }
            uint32_t mA = ((mA0 << 8) | mA1) & 0xFFFFu, mB = ((mB0 << 8) | mB1) & 0xFFFFu;
            if (EXACT && E == -__int_as_float(0x7f800000)) mA = mB = 0xFFFFu;  // re-check every centroid
            KTR(KTR_EPI, 16);
            const bool unique = __popc(mA) == 1 && __popc(mB) == 1;
            int bi = unique ? 16 * (15 - (31 - __clz(mB))) + (15 - (31 - __clz(mA))) : 0;
            if (__any_sync(0xffffffffu, !unique)) {  // warp-uniform
                if (!unique) {
                    float bd = __int_as_float(0x7f800000);
                    // the point's coordinates (global memory: the tile's stage may be recycled)
                    float xv[16];
                    const float4* xp = reinterpret_cast<const float4*>(xg + (valid ? p : p0) * 16);
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const float4 v = xp[j];
                        xv[4 * j] = v.x; xv[4 * j + 1] = v.y; xv[4 * j + 2] = v.z; xv[4 * j + 3] = v.w;
                    }
                    // 4-column groups of the product set, ascending (with the strict < the lowest
                    // index wins ties, as in the scalar loop): b-group lb, quarter qq of it
                    uint32_t quarters = 0;  // quarter k holds a-groups 4k..4k+3 (bits 15-4k..12-4k)
#pragma unroll
                    for (int k = 0; k < 4; ++k) quarters |= ((mA >> (12 - 4 * k)) & 0xFu) ? (1u << k) : 0u;
                    uint32_t mb = mB;
                    while (mb) {
                        const int lb = __clz(mb) - 16;  // bit 15 - lb
                        mb &= ~(0x8000u >> lb);
                        uint32_t qs = quarters;
                        while (qs) {
                            const int qq = __ffs(qs) - 1;
                            qs &= qs - 1;
                            const int G = 4 * lb + qq;  // 4-centroid group: centroids 16 lb + 4 qq ..
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
                    }
                }
            }
            KTR(KTR_EPI, 17);
            // member[] and the reductiontoarray count (the sums go through the MMA; a point whose
            // fixed-point values do not fit 16 bits adds them here, exact int64, to the partials)
            if (valid) {
                member[p] = bi;
                atomicAdd(&s_cnt[bi], 1);
                if (E < 0.f) {
                    const float4* xp = reinterpret_cast<const float4*>(xg + p * 16);
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const float4 v = xp[j];
                        const float e4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            if constexpr (EXACT) {
                                superacc_add_tc(reinterpret_cast<unsigned long long*>(sums) + (bi * 16 + 4 * j + e) * 9,
                                                e4[e]);
                            } else {
                                const float scale = (float)(1 << shift);
                                const long long iv = (long long)__float2int_rn(e4[e] * scale);
                                if (iv) atomicAdd(reinterpret_cast<unsigned long long*>(sums) + bi * 16 + 4 * j + e,
                                                  (unsigned long long)iv);
                            }
                        }
                    }
                }
            }
            // the point's one-hot byte (cluster row bi, point column r) in the set's stage; the
            // byte this thread set there two tiles ago is cleared first
            KPR(21, i);
            mbar_wait(&oempty[o], (uint32_t)((i / OS) & 1) ^ 1u);
            KTR(KTR_EPI, 19);
            if (pend >= 0) sts_u8(sOH + o * kOHBytes + (uint32_t)pend, 0u);
            pend = valid ? (int32_t)((uint32_t)(bi >> 7) * 16384u + sw_off((uint32_t)(bi & 127), (uint32_t)r)) : -1;
            if (valid) sts_u8(sOH + o * kOHBytes + (uint32_t)pend, 1u);
            fence_async_smem();
            mbar_arrive(&ofull[o]);
            KPR(22, i);
            KTR(KTR_EPI, 20);
        }
        // reduction accumulators: lane = cluster (h*128 + r), columns 2j+b = byte sums; counts
        // from the shared atomics (every epilogue warp has passed its last tile: named barrier)
        KPR(23, 0);
        named_bar(5, 256);
        KPR(24, 0);
        mbar_wait(sdone, 0);
        KPR(25, 0);
        tc_fence_after();
        for (int h = half; h < nh; h += 2) {
            uint32_t v0[32];
            const uint32_t tb2 = tq + kColSum + (uint32_t)(kRows * h);
            tmem_ld<32>(tb2, v0);
            tmem_wait();
            const int c = 128 * h + r;
            const uint64_t cnt = c < kc ? (uint64_t)s_cnt[c] : 0ull;
            if (cnt) {
#pragma unroll
                for (int j = 0; j < 16; ++j) {
                    const uint64_t su = (uint64_t)v0[2 * j] + ((uint64_t)v0[2 * j + 1] << 8);
                    const int64_t sv = (int64_t)(su - (cnt << 15));  // remove the 2^15 bias
                    if (sv) atomicAdd(reinterpret_cast<unsigned long long*>(sums) + c * 16 + j, (unsigned long long)sv);
                }
                atomicAdd(reinterpret_cast<unsigned long long*>(counts) + c, (unsigned long long)cnt);
            }
        }
    }
    tc_fence_before();
    KPR(26, 0);
    __syncthreads();
    KPR(27, 0);
    tc_fence_after();
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

}  // namespace

#ifdef KM_PROGRESS
static unsigned* h_prog = nullptr;
#endif
}  // namespace k
}  // namespace accmg
#ifdef KM_PROGRESS
// debug builds only: per-warp progress of the first 4096 CTAs in mapped host memory
extern "C" int accmg_km_progress_init(void) {
    if (cudaHostAlloc(&accmg::k::h_prog, 4096 * 16 * 4, cudaHostAllocMapped) != cudaSuccess) return -1;
    memset(accmg::k::h_prog, 0xff, 4096 * 16 * 4);
    unsigned* d = nullptr;
    cudaHostGetDevicePointer(&d, accmg::k::h_prog, 0);
    return cudaMemcpyToSymbol(accmg::k::g_prog, &d, sizeof(d)) == cudaSuccess ? 0 : -2;
}
extern "C" void accmg_km_progress_dump(int nctas) {
    for (int b = 0; b < nctas; ++b) {
        printf("cta %3d:", b);
        for (int w = 0; w < 16; ++w) printf(" %08x", accmg::k::h_prog[b * 16 + w]);
        printf("\n");
    }
    fflush(stdout);
}
#endif
namespace accmg {
namespace k {
namespace {
}  // namespace

int kmeans_tc_supported(const float* x, int d, int kc) {
    return d == 16 && kc >= 1 && kc <= KMAX && (reinterpret_cast<uintptr_t>(x) % 16) == 0;
}

cudaError_t kmeans_assign_tc(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                             int64_t p0, int64_t p1, int kc, int shift, int* err_flag, cudaStream_t s, int sms) {
    if (p1 <= p0) return cudaSuccess;
    if (p1 - p0 > (int64_t)INT32_MAX - TM) return cudaErrorNotSupported;  // TMA row coordinates are int32
    const int npad = ((kc + 31) / 32) * 32;
    const bool exact = shift < 0;  // ACCMG_KMEANS_EXACT
    cudaError_t e = exact ? kernel_prep(assign_tc<true>, kThreadsTC, kSmemTC) : kernel_prep(assign_tc<false>, kThreadsTC, kSmemTC);
    if (e != cudaSuccess) return e;
    const int64_t ntiles = (p1 - p0 + TM - 1) / TM;
    // s32 reduction accumulators: byte sums <= 255 per point, so at most 2^23 points (65536 tiles)
    // per CTA; more CTAs than SMs run in waves
    int64_t blocks = ntiles < sms ? ntiles : sms;
    const int64_t need = (ntiles + 65535) / 65536;
    if (blocks < need) blocks = need;
    // point tiles by TMA: [rows][16] fp32 from p0, 128-row boxes, 64-byte swizzle (the per-row
    // float4 reads of the converter and epilogue threads hit 8 distinct bank groups)
    CUtensorMap xmap;
    cuuint64_t dims[2] = {16, (cuuint64_t)(p1 - p0)};
    cuuint64_t strides[1] = {64};
    cuuint32_t box[2] = {16, TM};
    cuuint32_t es[2] = {1, 1};
    if (!tma_encode_tiled(&xmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(x) + p0 * 16, dims, strides,
                          box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
                          CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE))
        return cudaErrorNotSupported;
    if (exact)
        assign_tc<true><<<(unsigned)blocks, kThreadsTC, kSmemTC, s>>>(xmap, x, cen, member, sums, counts, p0, p1, kc, npad,
                                                                     shift, err_flag);
    else
        assign_tc<false><<<(unsigned)blocks, kThreadsTC, kSmemTC, s>>>(xmap, x, cen, member, sums, counts, p0, p1, kc, npad, shift,
                                                            err_flag);
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
