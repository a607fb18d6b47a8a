// Loop bodies of the k-means workload (config C4; KMEANS is the paper's Rodinia application,
// Table II, with 2 parallel loops and a reductiontoarray, L75-77/L89-91/L112).
//
// Assignment loop over points p (this partition's chunk):
//   best = 0, bestd = +inf; for c: acc = 0; for j: diff = x[p][j] - cen[c][j]; acc = fmaf(diff, diff, acc);
//   if (acc < bestd) {bestd = acc; best = c}      (ties -> lowest c; reading in DESIGN.md)
//   member[p] = best;  sums[best][j] += x[p][j] (exact: int64 fixed point x*2^shift);  counts[best] += 1
// Hierarchical reduction (L112): shared-memory accumulators per block, then one global atomic per
// non-zero entry into the partition's partial, then (runtime) across partitions / GPUs.
//
// FP32-pipe bound (2*k*d flops per point, no tensor-core form preserves the exact fmaf order that
// the bit-exact argmin needs). Two points share each packed __fadd2_rn / __ffma2_rn
// (Blackwell FADD2/FFMA2: two fp32 lanes per instruction, each rounded exactly like the scalar op),
// so the per-distance operation order is the scalar one; each thread owns 4 points; centroids
// are staged in shared memory pre-negated and duplicated as float2 (-c, -c) so one LDS.128 feeds
// two dims of two packed pairs, and the next centroid is prefetched while the current one is
// consumed. Packed ops halve the issue slots but not the FP32 lane rate (128 lanes/clk/SM,
// measured with scripts/fp32_micro.cu), which is the roofline of this kernel.
#include <cstdlib>

#include "kernels.h"
#include "tma_host.h"
#include "track.cuh"

namespace accmg {
namespace k {
namespace {

constexpr int kThreads = 256;

__device__ __forceinline__ int64_t fixed_of(float x, float scale, int* err) {
    const float v = x * scale;  // exact: power-of-two scaling
    if (!(v == rintf(v) && fabsf(v) < 2147483648.0f)) atomicOr(err, 1);
    return (int64_t)v;
}

// Packed fp32x2 arithmetic on 64-bit registers (PTX add/fma .f32x2, sm_100): each lane is
// rounded exactly like the scalar add.rn / fma.rn. Holding the pairs as .b64 values keeps them in
// aligned register pairs (the float2 builtins let ptxas re-pair scalars with MOVs every use).
__device__ __forceinline__ uint64_t pk2(float a, float b) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
// Materialises a pair in an aligned register pair: x + (-0) == x for every x (also +-0), done
// by a real FADD2 so the allocator keeps the pair instead of re-pairing scalars on every use.
__device__ __forceinline__ uint64_t pk2m(float a, float b) {
    uint64_t r;
    asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(pk2(a, b)), "l"(0x8000000080000000ull));
    return r;
}
__device__ __forceinline__ void upk2(uint64_t v, float& a, float& b) {
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
__device__ __forceinline__ uint64_t add2(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ uint64_t fma2sq(uint64_t d, uint64_t acc) {  // d*d + acc
    uint64_t r;
    asm("fma.rn.f32x2 %0, %1, %1, %2;" : "=l"(r) : "l"(d), "l"(acc));
    return r;
}

// Block-level accumulation into shared memory, then flush to the partition's partial (global).
__device__ __forceinline__ void flush_block(unsigned long long* s_sum, unsigned long long* s_cnt, int64_t* sums,
                                            int64_t* counts, int kc, int d) {
    __syncthreads();
    for (int i = threadIdx.x; i < kc * d; i += blockDim.x)
        if (s_sum[i]) atomicAdd(reinterpret_cast<unsigned long long*>(sums) + i, s_sum[i]);
    for (int i = threadIdx.x; i < kc; i += blockDim.x)
        if (s_cnt[i]) atomicAdd(reinterpret_cast<unsigned long long*>(counts) + i, s_cnt[i]);
}

// D dims, NP packed point pairs per thread (2*NP points), CU centroids per step (NP*CU
// independent FFMA2 chains per thread hide the packed-op latency; one LDS.128 of a centroid's
// duplicated pair of dims feeds 4*NP packed operations).
template <int D, int NP, int CU, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB)
assign_d(const float* __restrict__ x, const float* __restrict__ cen, int32_t* __restrict__ member,
         int64_t* __restrict__ sums, int64_t* __restrict__ counts, int64_t p0, int64_t p1, int kc, int shift,
         int* err) {
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned long long* s_sum = reinterpret_cast<unsigned long long*>(smem);           // kc*D
    unsigned long long* s_cnt = s_sum + kc * D;                                      // kc
    float* s_nc = reinterpret_cast<float*>(s_cnt + kc);                              // kc*D  (-c)
    for (int i = threadIdx.x; i < kc * D; i += NT) {
        s_nc[i] = -cen[i];
        s_sum[i] = 0ull;
    }
    for (int i = threadIdx.x; i < kc; i += NT) s_cnt[i] = 0ull;
    __syncthreads();
    constexpr int PPT = 2 * NP;
    const float scale = (float)(1 << shift);
    const int64_t n = p1 - p0;
    const int64_t ngroups = (n + PPT - 1) / PPT;
    for (int64_t grp = (int64_t)blockIdx.x * NT + threadIdx.x; grp < ngroups; grp += (int64_t)gridDim.x * NT) {
        const int64_t pb = p0 + grp * PPT;
        uint64_t xp[NP][D];  // pair h = (x[pb+2h][j], x[pb+2h+1][j])
#pragma unroll
        for (int h = 0; h < NP; ++h) {
            const bool ok0 = pb + 2 * h < p1, ok1 = pb + 2 * h + 1 < p1;
#pragma unroll
            for (int j = 0; j < D; j += 4) {
                const float4 a = ok0 ? __ldg(reinterpret_cast<const float4*>(x + (pb + 2 * h) * D + j))
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
                const float4 b = ok1 ? __ldg(reinterpret_cast<const float4*>(x + (pb + 2 * h + 1) * D + j))
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
                xp[h][j] = pk2m(a.x, b.x);
                xp[h][j + 1] = pk2m(a.y, b.y);
                xp[h][j + 2] = pk2m(a.z, b.z);
                xp[h][j + 3] = pk2m(a.w, b.w);
            }
        }
        float bd[PPT];
        int bi[PPT];
#pragma unroll
        for (int q = 0; q < PPT; ++q) { bd[q] = __int_as_float(0x7f800000); bi[q] = 0; }
        const float4* nc4 = reinterpret_cast<const float4*>(s_nc);
        // the next centroid group's values are loaded while the current one is consumed (the
        // shared-memory latency is off the critical path); one LDS.128 brings 4 dims, and FADD2
        // takes each dim as a scalar operand broadcast to both lanes
        float4 ncur[CU][D / 4];
#pragma unroll
        for (int u = 0; u < CU; ++u)
#pragma unroll
            for (int jj = 0; jj < D / 4; ++jj) ncur[u][jj] = nc4[(u * D) / 4 + jj];
#pragma unroll 1
        for (int c = 0; c < kc; c += CU) {
            float4 nnext[CU][D / 4];
            const int cn = (c + CU < kc) ? c + CU : c;
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int jj = 0; jj < D / 4; ++jj) nnext[u][jj] = nc4[((cn + u) * D) / 4 + jj];
            uint64_t acc[CU][NP];
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int h = 0; h < NP; ++h) acc[u][h] = 0ull;
#pragma unroll
            for (int j = 0; j < D; ++j) {
#pragma unroll
                for (int u = 0; u < CU; ++u) {
                    const float4 q4 = ncur[u][j / 4];
                    const float nj = (j % 4 == 0) ? q4.x : (j % 4 == 1) ? q4.y : (j % 4 == 2) ? q4.z : q4.w;
                    const uint64_t n2 = pk2(nj, nj);
#pragma unroll
                    for (int h = 0; h < NP; ++h) acc[u][h] = fma2sq(add2(xp[h][j], n2), acc[u][h]);
                }
            }
            // centroids in ascending order: strict < keeps the lowest index on ties
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int h = 0; h < NP; ++h) {
                    float d0, d1;
                    upk2(acc[u][h], d0, d1);
                    if (d0 < bd[2 * h]) { bd[2 * h] = d0; bi[2 * h] = c + u; }
                    if (d1 < bd[2 * h + 1]) { bd[2 * h + 1] = d1; bi[2 * h + 1] = c + u; }
                }
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int jj = 0; jj < D / 4; ++jj) ncur[u][jj] = nnext[u][jj];
        }
#pragma unroll
        for (int q = 0; q < PPT; ++q) {
            if (pb + q >= p1) continue;
            member[pb + q] = bi[q];
            atomicAdd(s_cnt + bi[q], 1ull);
#pragma unroll
            for (int j = 0; j < D; ++j) {
                float xa, xb;
                upk2(xp[q / 2][j], xa, xb);
                const float xv = (q & 1) ? xb : xa;
                atomicAdd(s_sum + bi[q] * D + j, (unsigned long long)fixed_of(xv, scale, err));
            }
        }
    }
    flush_block(s_sum, s_cnt, sums, counts, kc, D);
}

// Centroids in constant memory (default for d = 16, k <= kConstCen): the loop over c is
// warp-uniform, so the compiler reads each centroid value with a uniform-datapath LDCU into a
// uniform register and FADD2 takes it as a broadcast scalar operand with a free negation
// (`FADD2 R, R.F32x2, -UR.F32`: x + (-c) == x - c exactly). No shared-memory loads on the vector
// pipes and no centroid copies in vector registers (108 instead of 125 registers at 2 blocks/SM).
// The loop over this thread's point groups takes its trip count from block-uniform values only:
// with a per-thread grid-stride condition the compiler cannot prove the centroid loop convergent
// and falls back to vector LDC loads (measured: 8 % slower).
constexpr int kConstCen = 512;
__constant__ float c_cen[kConstCen * 16];

template <int NP, int CU, int NT, int MINB, int UNR = 1>
__global__ void __launch_bounds__(NT, MINB)
assign_c16(const float* __restrict__ x, int32_t* __restrict__ member, int64_t* __restrict__ sums,
           int64_t* __restrict__ counts, int64_t p0, int64_t p1, int kc, int shift, int* err) {
    constexpr int D = 16;
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned long long* s_sum = reinterpret_cast<unsigned long long*>(smem);  // kc*D
    unsigned long long* s_cnt = s_sum + kc * D;                             // kc
    for (int i = threadIdx.x; i < kc * D; i += NT) s_sum[i] = 0ull;
    for (int i = threadIdx.x; i < kc; i += NT) s_cnt[i] = 0ull;
    __syncthreads();
    constexpr int PPT = 2 * NP;
    const float scale = (float)(1 << shift);
    const int64_t n = p1 - p0;
    const int64_t ngroups = (n + PPT - 1) / PPT;
    // trip count from block-uniform values only, so the centroid loop below runs under uniform
    // control flow (the condition for the uniform-datapath LDCU of c_cen); lanes past the end
    // compute on zeros and store nothing
    const int64_t first = (int64_t)blockIdx.x * NT, stride = (int64_t)gridDim.x * NT;
    const int64_t trips = first < ngroups ? (ngroups - first + stride - 1) / stride : 0;
    for (int64_t it = 0; it < trips; ++it) {
        const int64_t grp = first + it * stride + threadIdx.x;
        const int64_t pb = p0 + grp * PPT;
        uint64_t xp[NP][D];  // pair h = (x[pb+2h][j], x[pb+2h+1][j])
#pragma unroll
        for (int h = 0; h < NP; ++h) {
            const bool ok0 = pb + 2 * h < p1, ok1 = pb + 2 * h + 1 < p1;
#pragma unroll
            for (int j = 0; j < D; j += 4) {
                const float4 a = ok0 ? __ldg(reinterpret_cast<const float4*>(x + (pb + 2 * h) * D + j))
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
                const float4 b = ok1 ? __ldg(reinterpret_cast<const float4*>(x + (pb + 2 * h + 1) * D + j))
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
                xp[h][j] = pk2m(a.x, b.x);
                xp[h][j + 1] = pk2m(a.y, b.y);
                xp[h][j + 2] = pk2m(a.z, b.z);
                xp[h][j + 3] = pk2m(a.w, b.w);
            }
        }
        float bd[PPT];
        int bi[PPT];
#pragma unroll
        for (int q = 0; q < PPT; ++q) { bd[q] = __int_as_float(0x7f800000); bi[q] = 0; }
#pragma unroll UNR
        for (int c = 0; c < kc; c += CU) {
            uint64_t acc[CU][NP];
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int h = 0; h < NP; ++h) acc[u][h] = 0ull;
#pragma unroll
            for (int j = 0; j < D; ++j) {
#pragma unroll
                for (int u = 0; u < CU; ++u) {
                    const float nj = -c_cen[(c + u) * D + j];
                    const uint64_t n2 = pk2(nj, nj);
#pragma unroll
                    for (int h = 0; h < NP; ++h) acc[u][h] = fma2sq(add2(xp[h][j], n2), acc[u][h]);
                }
            }
            // centroids in ascending order: strict < keeps the lowest index on ties
#pragma unroll
            for (int u = 0; u < CU; ++u)
#pragma unroll
                for (int h = 0; h < NP; ++h) {
                    float d0, d1;
                    upk2(acc[u][h], d0, d1);
                    if (d0 < bd[2 * h]) { bd[2 * h] = d0; bi[2 * h] = c + u; }
                    if (d1 < bd[2 * h + 1]) { bd[2 * h + 1] = d1; bi[2 * h + 1] = c + u; }
                }
        }
#pragma unroll
        for (int q = 0; q < PPT; ++q) {
            if (pb + q >= p1) continue;
            member[pb + q] = bi[q];
            atomicAdd(s_cnt + bi[q], 1ull);
#pragma unroll
            for (int j = 0; j < D; ++j) {
                float xa, xb;
                upk2(xp[q / 2][j], xa, xb);
                const float xv = (q & 1) ? xb : xa;
                atomicAdd(s_sum + bi[q] * D + j, (unsigned long long)fixed_of(xv, scale, err));
            }
        }
    }
    flush_block(s_sum, s_cnt, sums, counts, kc, D);
}

template <int NP, int CU, int NT, int MINB, int UNR = 1>
cudaError_t launch_assign_c16(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                              int64_t p0, int64_t p1, int kc, int shift, int* err, cudaStream_t s, int sms) {
    auto kern = assign_c16<NP, CU, NT, MINB, UNR>;
    cudaError_t e = cudaMemcpyToSymbolAsync(c_cen, cen, (size_t)kc * 16 * sizeof(float), 0, cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) return e;
    const size_t smem = (size_t)kc * 16 * 8 + (size_t)kc * 8;
    int per_sm = 0;
    e = kernel_prep(kern, NT, smem, &per_sm);
    if (e != cudaSuccess) return e;
    const int64_t groups = (p1 - p0 + 2 * NP - 1) / (2 * NP);
    int64_t blocks = (groups + NT - 1) / NT;
    const int64_t cap = (int64_t)sms * (per_sm > 0 ? per_sm : 1);
    if (blocks > cap) blocks = cap;
    kern<<<(unsigned)blocks, NT, smem, s>>>(x, member, sums, counts, p0, p1, kc, shift, err);
    return cudaGetLastError();
}

template <int NP, int CU, int NT, int MINB = 1>
cudaError_t launch_assign16(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                            int64_t p0, int64_t p1, int kc, int shift, int* err, cudaStream_t s, int sms) {
    auto kern = assign_d<16, NP, CU, NT, MINB>;
    const size_t smem = (size_t)kc * 16 * 8 + (size_t)kc * 8 + (size_t)kc * 16 * 4;
    if (smem > 200 * 1024) return cudaErrorNotSupported;
    // all of the unified L1/shared capacity as shared memory, so several blocks fit per SM
    int per_sm = 0;
    cudaError_t e = kernel_prep(kern, NT, smem, &per_sm, true);
    if (e != cudaSuccess) return e;
    const int64_t groups = (p1 - p0 + 2 * NP - 1) / (2 * NP);
    int64_t blocks = (groups + NT - 1) / NT;
    const int64_t cap = (int64_t)sms * (per_sm > 0 ? per_sm : 1);
    if (blocks > cap) blocks = cap;
    kern<<<(unsigned)blocks, NT, smem, s>>>(x, cen, member, sums, counts, p0, p1, kc, shift, err);
    return cudaGetLastError();
}

// Generic d (any d <= 32): one point per thread, scalar fmaf chain in the same order.
__global__ void __launch_bounds__(kThreads)
assign_generic(const float* __restrict__ x, const float* __restrict__ cen, int32_t* __restrict__ member,
               int64_t* __restrict__ sums, int64_t* __restrict__ counts, int64_t p0, int64_t p1, int d, int kc,
               int shift, int* err) {
    extern __shared__ __align__(16) unsigned char smem[];
    float* s_c = reinterpret_cast<float*>(smem);
    unsigned long long* s_sum = reinterpret_cast<unsigned long long*>(smem + ((kc * d * 4 + 15) / 16) * 16);
    unsigned long long* s_cnt = s_sum + kc * d;
    for (int i = threadIdx.x; i < kc * d; i += kThreads) { s_c[i] = cen[i]; s_sum[i] = 0ull; }
    for (int i = threadIdx.x; i < kc; i += kThreads) s_cnt[i] = 0ull;
    __syncthreads();
    const float scale = (float)(1 << shift);
    for (int64_t p = p0 + (int64_t)blockIdx.x * kThreads + threadIdx.x; p < p1; p += (int64_t)gridDim.x * kThreads) {
        float xv[32];
        for (int j = 0; j < d; ++j) xv[j] = x[p * d + j];
        float bd = __int_as_float(0x7f800000);
        int bi = 0;
        for (int c = 0; c < kc; ++c) {
            float acc = 0.f;
            for (int j = 0; j < d; ++j) {
                const float df = __fsub_rn(xv[j], s_c[c * d + j]);
                acc = __fmaf_rn(df, df, acc);
            }
            if (acc < bd) { bd = acc; bi = c; }
        }
        member[p] = bi;
        atomicAdd(s_cnt + bi, 1ull);
        for (int j = 0; j < d; ++j) atomicAdd(s_sum + bi * d + j, (unsigned long long)fixed_of(xv[j], scale, err));
    }
    flush_block(s_sum, s_cnt, sums, counts, kc, d);
}

// Update loop, element pass: e = c*d + j over clusters [c0, c1):
//   if counts[c] > 0: cen[e] = (float)(((double)sums[e] * 2^-shift) / (double)counts[c]);  sums[e] = 0.
template <bool TRACK>
__global__ void __launch_bounds__(kThreads)
update_elems(int64_t* __restrict__ sums, const int64_t* __restrict__ counts, float* __restrict__ cen, int64_t c0,
             int64_t c1, int d, int shift, Track ts, Track tc) {
    const int64_t e0 = c0 * d, e1 = c1 * d;
    const double inv = 1.0 / (double)(1ll << shift);  // exact power of two
    int64_t cs = -1, cc = -1;
    for (int64_t base = e0 + (int64_t)blockIdx.x * kThreads; base < e1; base += (int64_t)gridDim.x * kThreads) {
        const int64_t e = base + threadIdx.x;
        const bool ok = e < e1;
        bool wc = false;
        if (ok) {
            const int64_t c = e / d;
            const int64_t cnt = counts[c];
            if (cnt > 0) {
                cen[e] = (float)(__dmul_rn((double)sums[e], inv) / (double)cnt);
                wc = true;
            }
            sums[e] = 0;
        }
        if constexpr (TRACK) {
            const int64_t wb = base + (threadIdx.x & ~31);
            if (ts.l1) dev::track_warp<1>(ts.l1, ts.l2, ts.l2_shift, wb, ok ? 1u : 0u, cs);
            if (tc.l1) dev::track_warp<1>(tc.l1, tc.l2, tc.l2_shift, wb, wc ? 1u : 0u, cc);
        }
    }
}

// Update loop, cluster pass: counts[c] = 0 for c in [c0, c1) (after the element pass read them).
template <bool TRACK>
__global__ void __launch_bounds__(kThreads)
update_counts(int64_t* __restrict__ counts, int64_t c0, int64_t c1, Track t) {
    int64_t l2c = -1;
    for (int64_t base = c0 + (int64_t)blockIdx.x * kThreads; base < c1; base += (int64_t)gridDim.x * kThreads) {
        const int64_t c = base + threadIdx.x;
        if (c < c1) counts[c] = 0;
        if constexpr (TRACK) {
            if (t.l1) dev::track_warp<1>(t.l1, t.l2, t.l2_shift, base + (threadIdx.x & ~31), c < c1 ? 1u : 0u, l2c);
        }
    }
}

// ---- exact mode (args.shift = -1): arbitrary finite fp32 points (reading KM-X in DESIGN.md) -----
// The centroid update needs RN64(exact sum of the members' values): each value x = m * 2^(o - 149)
// (m the 24-bit significand, o = biased exponent - 1, or 0 for subnormals) is added exactly into
// nine 32-bit-aligned windows, A_w of weight 2^(32 w - 149): m * 2^(o mod 32) < 2^55 splits into a
// low 32-bit part for window o / 32 and a high part for the next one. Every addend is below 2^32
// in magnitude, so an int64 window holds the sum of up to 2^31 of them exactly; the sums region
// holds k * d * 9 such windows (REDUCE_SUM merges them elementwise like any int64 partials).
constexpr int kSuperW = 9;

__device__ __forceinline__ void superacc_add(unsigned long long* acc, float v, int* err) {
    const uint32_t b = __float_as_uint(v);
    const uint32_t ex = (b >> 23) & 255u;
    if (ex == 255u) {  // inf / NaN: no exact mean
        atomicOr(err, 1);
        return;
    }
    uint32_t m = b & 0x7FFFFFu;
    if (ex) m |= 0x800000u;
    if (!m) return;
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

// Assignment (the scalar loop, any data) + exact reductiontoarray into the windows. DM >= d: the
// points live in registers, NPT points per thread share every centroid load (rows padded to a
// multiple of 4 floats in shared memory, one LDS.128 per 4 dims). Windows and counts in shared
// memory when they fit (flushed once per block), else straight into the partition's partials.
template <int DM, int NPT, bool SHARED_ACC>
__global__ void __launch_bounds__(kThreads)
assign_exact_k(const float* __restrict__ x, const float* __restrict__ cen, int32_t* __restrict__ member,
               int64_t* __restrict__ sacc, int64_t* __restrict__ counts, int64_t p0, int64_t p1, int d, int kc,
               int* err) {
    extern __shared__ __align__(16) unsigned char smem_e[];
    const int dp = (d + 3) & ~3;  // padded centroid row
    float4* s_c4 = reinterpret_cast<float4*>(smem_e);
    float* s_c = reinterpret_cast<float*>(smem_e);
    unsigned long long* s_cnt = reinterpret_cast<unsigned long long*>(smem_e + (size_t)kc * dp * 4);
    unsigned long long* s_acc = s_cnt + kc;
    for (int i = threadIdx.x; i < kc * dp; i += blockDim.x) {
        const int c = i / dp, j = i - c * dp;
        s_c[i] = j < d ? cen[c * d + j] : 0.f;
    }
    for (int i = threadIdx.x; i < kc; i += blockDim.x) s_cnt[i] = 0ull;
    if constexpr (SHARED_ACC)
        for (int i = threadIdx.x; i < kc * d * kSuperW; i += blockDim.x) s_acc[i] = 0ull;
    __syncthreads();
    unsigned long long* acc = SHARED_ACC ? s_acc : reinterpret_cast<unsigned long long*>(sacc);
    const int64_t step = (int64_t)gridDim.x * blockDim.x * NPT;
    for (int64_t pb = p0 + (int64_t)blockIdx.x * blockDim.x * NPT + threadIdx.x; pb < p1; pb += step) {
        float xv[NPT][DM];
#pragma unroll
        for (int q = 0; q < NPT; ++q) {
            const int64_t p = pb + (int64_t)q * blockDim.x;
#pragma unroll
            for (int j = 0; j < DM; ++j) xv[q][j] = (j < d && p < p1) ? x[p * d + j] : 0.f;
        }
        float bd[NPT];
        int bi[NPT];
#pragma unroll
        for (int q = 0; q < NPT; ++q) { bd[q] = __int_as_float(0x7f800000); bi[q] = 0; }
        for (int c = 0; c < kc; ++c) {
            float a[NPT];
#pragma unroll
            for (int q = 0; q < NPT; ++q) a[q] = 0.f;
#pragma unroll
            for (int j4 = 0; j4 < DM / 4; ++j4)
                if (4 * j4 < d) {
                    const float4 cv = s_c4[c * (dp >> 2) + j4];
                    const float ce[4] = {cv.x, cv.y, cv.z, cv.w};
#pragma unroll
                    for (int e = 0; e < 4; ++e)
                        if (4 * j4 + e < d) {
#pragma unroll
                            for (int q = 0; q < NPT; ++q) {
                                const float df = __fsub_rn(xv[q][4 * j4 + e], ce[e]);
                                a[q] = __fmaf_rn(df, df, a[q]);
                            }
                        }
                }
#pragma unroll
            for (int q = 0; q < NPT; ++q)
                if (a[q] < bd[q]) { bd[q] = a[q]; bi[q] = c; }
        }
#pragma unroll
        for (int q = 0; q < NPT; ++q) {
            const int64_t p = pb + (int64_t)q * blockDim.x;
            if (p >= p1) continue;
            member[p] = bi[q];
            atomicAdd(s_cnt + bi[q], 1ull);
#pragma unroll
            for (int j = 0; j < DM; ++j)
                if (j < d) superacc_add(acc + ((size_t)bi[q] * d + j) * kSuperW, xv[q][j], err);
        }
    }
    __syncthreads();
    if constexpr (SHARED_ACC)
        for (int i = threadIdx.x; i < kc * d * kSuperW; i += blockDim.x)
            if (s_acc[i]) atomicAdd(reinterpret_cast<unsigned long long*>(sacc) + i, s_acc[i]);
    for (int i = threadIdx.x; i < kc; i += blockDim.x)
        if (s_cnt[i]) atomicAdd(reinterpret_cast<unsigned long long*>(counts) + i, s_cnt[i]);
}

// RN64 of sum_w A[w] * 2^(32 w - 149): carry-normalise to base-2^32 digits (two's complement over
// ten digits), take the magnitude, round its leading 96 bits to 53 with a sticky bit for the rest
// (ties to even). The exact sum of fp32 values is 0 or of magnitude in [2^-149, 2^160): a normal
// double, so the scaling is exact.
__device__ double superacc_round(const int64_t* __restrict__ A) {
    uint32_t dg[kSuperW + 1];
    long long carry = 0;
#pragma unroll
    for (int w = 0; w < kSuperW; ++w) {
        const __int128 t = (__int128)A[w] + carry;
        dg[w] = (uint32_t)(unsigned long long)t;
        carry = (long long)(t >> 32);
    }
    dg[kSuperW] = (uint32_t)carry;
    const bool neg = carry < 0;
    if (neg) {  // magnitude: invert and add one
        unsigned long long c1 = 1ull;
#pragma unroll
        for (int w = 0; w <= kSuperW; ++w) {
            const unsigned long long t = (unsigned long long)(uint32_t)~dg[w] + c1;
            dg[w] = (uint32_t)t;
            c1 = t >> 32;
        }
    }
    int top = -1;
#pragma unroll
    for (int w = 0; w <= kSuperW; ++w)
        if (dg[w]) top = w;
    if (top < 0) return 0.0;
    uint32_t d1 = 0u, d2 = 0u;
    bool sticky = false;
#pragma unroll
    for (int w = 0; w <= kSuperW; ++w) {
        if (w == top - 1) d1 = dg[w];
        if (w == top - 2) d2 = dg[w];
        if (w < top - 2 && dg[w]) sticky = true;
    }
    const unsigned __int128 M = ((unsigned __int128)dg[top] << 64) | ((unsigned __int128)d1 << 32) | d2;
    const int lead = 95 - __clz(dg[top]);  // leading bit of M
    const int sh = lead - 52;              // 12..43
    unsigned long long mant = (unsigned long long)(M >> sh);
    const unsigned __int128 rem = M & ((((unsigned __int128)1) << sh) - 1);
    const unsigned __int128 half = ((unsigned __int128)1) << (sh - 1);
    if (rem > half || (rem == half && (sticky || (mant & 1ull)))) ++mant;  // 2^53 stays exact
    const double r = ldexp((double)mant, sh + 32 * (top - 2) - 149);
    return neg ? -r : r;
}

// Update, element pass (exact mode): if counts[c] > 0: cen[e] = (float)(RN64(sum) / counts[c]).
template <bool TRACK>
__global__ void __launch_bounds__(kThreads)
update_exact_elems(const int64_t* __restrict__ sacc, const int64_t* __restrict__ counts, float* __restrict__ cen,
                   int64_t c0, int64_t c1, int d, Track tc) {
    const int64_t e0 = c0 * d, e1 = c1 * d;
    int64_t cc = -1;
    for (int64_t base = e0 + (int64_t)blockIdx.x * kThreads; base < e1; base += (int64_t)gridDim.x * kThreads) {
        const int64_t e = base + threadIdx.x;
        bool wc = false;
        if (e < e1) {
            const int64_t cnt = counts[e / d];
            if (cnt > 0) {
                cen[e] = __double2float_rn(__ddiv_rn(superacc_round(sacc + e * kSuperW), (double)cnt));
                wc = true;
            }
        }
        if constexpr (TRACK) {
            if (tc.l1) dev::track_warp<1>(tc.l1, tc.l2, tc.l2_shift, base + (threadIdx.x & ~31), wc ? 1u : 0u, cc);
        }
    }
}

// Update, window pass (exact mode): sums[q] = 0 for the windows of clusters [c0, c1).
template <bool TRACK>
__global__ void __launch_bounds__(kThreads)
update_exact_zero(int64_t* __restrict__ sacc, int64_t q0, int64_t q1, Track ts) {
    int64_t cs = -1;
    for (int64_t base = q0 + (int64_t)blockIdx.x * kThreads; base < q1; base += (int64_t)gridDim.x * kThreads) {
        const int64_t q = base + threadIdx.x;
        if (q < q1) sacc[q] = 0;
        if constexpr (TRACK) {
            if (ts.l1) dev::track_warp<1>(ts.l1, ts.l2, ts.l2_shift, base + (threadIdx.x & ~31), q < q1 ? 1u : 0u, cs);
        }
    }
}

template <int DM>
cudaError_t launch_assign_exact(const float* x, const float* cen, int32_t* member, int64_t* sacc, int64_t* counts,
                                int64_t p0, int64_t p1, int d, int kc, int* err, cudaStream_t s, int sms) {
    constexpr int NPT = DM <= 16 ? 4 : DM <= 32 ? 2 : 1;
    const size_t base = (size_t)kc * ((d + 3) & ~3) * 4 + (size_t)kc * 8;
    const size_t shared_acc = base + (size_t)kc * d * kSuperW * 8;
    const bool sh = shared_acc <= 160 * 1024;
    const size_t smem = sh ? shared_acc : base;
    const void* fn = sh ? (const void*)assign_exact_k<DM, NPT, true> : (const void*)assign_exact_k<DM, NPT, false>;
    cudaError_t e = sh ? kernel_prep(assign_exact_k<DM, NPT, true>, kThreads, smem)
                       : kernel_prep(assign_exact_k<DM, NPT, false>, kThreads, smem);
    if (e != cudaSuccess) return e;
    int per_sm = 1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kThreads, smem);
    if (per_sm < 1) per_sm = 1;
    int64_t blocks = (p1 - p0 + kThreads * NPT - 1) / (kThreads * NPT);
    if (blocks > (int64_t)sms * per_sm) blocks = (int64_t)sms * per_sm;
    if (sh)
        assign_exact_k<DM, NPT, true><<<(unsigned)blocks, kThreads, smem, s>>>(x, cen, member, sacc, counts, p0, p1, d, kc, err);
    else
        assign_exact_k<DM, NPT, false><<<(unsigned)blocks, kThreads, smem, s>>>(x, cen, member, sacc, counts, p0, p1, d, kc, err);
    return cudaGetLastError();
}

int sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

}  // namespace

cudaError_t kmeans_assign(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                          int64_t p0, int64_t p1, int d, int kc, int shift, int* err_flag, cudaStream_t s,
                          int64_t* launches) {
    if (p1 <= p0) return cudaSuccess;
    const int sms = sm_count();
    if (shift < 0) {  // exact mode (arbitrary finite points; sums = k * d * 9 windows)
        if (kmeans_tc_supported(x, d, kc)) {  // d = 16, k <= 256: the tensor-core filter serves it too
            cudaError_t e = kmeans_assign_tc(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms);
            if (e == cudaSuccess) {
                if (launches) *launches += 1;
                return cudaSuccess;
            }
            if (e != cudaErrorNotSupported) return e;
            (void)cudaGetLastError();
        }
        if (d > 64 || (int64_t)kc * d > 16384) return cudaErrorNotSupported;
        cudaError_t e = d <= 16   ? launch_assign_exact<16>(x, cen, member, sums, counts, p0, p1, d, kc, err_flag, s, sms)
                        : d <= 32 ? launch_assign_exact<32>(x, cen, member, sums, counts, p0, p1, d, kc, err_flag, s, sms)
                                  : launch_assign_exact<64>(x, cen, member, sums, counts, p0, p1, d, kc, err_flag, s, sms);
        if (e == cudaSuccess && launches) *launches += 1;
        return e;
    }
    // the tensor-core filter + exact re-check (kmeans_tc.cu) where supported (d = 16, k <= 256);
    // the FP32-pipe kernels below otherwise
    if (kmeans_tc_supported(x, d, kc)) {
        cudaError_t e = kmeans_assign_tc(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms);
        if (e == cudaSuccess) {
            if (launches) *launches += 1;
            return cudaSuccess;
        }
        if (e != cudaErrorNotSupported) return e;
        (void)cudaGetLastError();  // unsupported shape for the tensor-core kernel: FP32-pipe kernels below
    }
    if (d == 16 && (reinterpret_cast<uintptr_t>(x) % 16) == 0) {
        // centroids in constant memory when they fit (kc <= kConstCen), else the shared-memory
        // kernel; measured on B200 (profiles/r01/kmeans_variants.txt): 3 blocks/SM (24 warps;
        // ptxas keeps 80 registers + 24 B of spills outside the centroid loop): 21.05 ms vs 21.43
        // for 2 blocks/SM
        cudaError_t e;
        const bool cu2 = kc % 2 == 0;
        if (kc <= kConstCen)
            e = cu2 ? launch_assign_c16<2, 2, 256, 3>(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms)
                    : launch_assign_c16<2, 1, 256, 3>(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms);
        else
            e = cu2 ? launch_assign16<2, 2, 256, 2>(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms)
                    : launch_assign16<2, 1, 256, 2>(x, cen, member, sums, counts, p0, p1, kc, shift, err_flag, s, sms);
        if (e != cudaSuccess) return e;
    } else {
        const size_t smem = (((size_t)kc * d * 4 + 15) / 16) * 16 + (size_t)kc * d * 8 + (size_t)kc * 8;
        if (smem > 200 * 1024) return cudaErrorNotSupported;
        cudaError_t e = kernel_prep(assign_generic, kThreads, smem);
        if (e != cudaSuccess) return e;
        int64_t blocks = (p1 - p0 + kThreads - 1) / kThreads;
        if (blocks > (int64_t)sms * 4) blocks = (int64_t)sms * 4;
        assign_generic<<<(unsigned)blocks, kThreads, smem, s>>>(x, cen, member, sums, counts, p0, p1, d, kc, shift, err_flag);
    }
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t kmeans_update(int64_t* sums, int64_t* counts, float* cen, int64_t c0, int64_t c1, int d, int shift,
                          Track t_sums, Track t_counts, Track t_cen, cudaStream_t s, int64_t* launches) {
    if (c1 <= c0) return cudaSuccess;
    const bool tr = t_sums.l1 || t_cen.l1;
    int64_t nb = ((c1 - c0) * d + kThreads - 1) / kThreads;
    if (nb > 1184) nb = 1184;
    if (shift < 0) {  // exact mode: the element pass reads all windows before the window pass clears them
        if (t_cen.l1) update_exact_elems<true><<<(unsigned)nb, kThreads, 0, s>>>(sums, counts, cen, c0, c1, d, t_cen);
        else update_exact_elems<false><<<(unsigned)nb, kThreads, 0, s>>>(sums, counts, cen, c0, c1, d, t_cen);
        const int64_t q0 = c0 * d * kSuperW, q1 = c1 * d * kSuperW;
        int64_t nq = (q1 - q0 + kThreads - 1) / kThreads;
        if (nq > 1184) nq = 1184;
        if (t_sums.l1) update_exact_zero<true><<<(unsigned)nq, kThreads, 0, s>>>(sums, q0, q1, t_sums);
        else update_exact_zero<false><<<(unsigned)nq, kThreads, 0, s>>>(sums, q0, q1, t_sums);
        int64_t nc = (c1 - c0 + kThreads - 1) / kThreads;
        if (nc > 1184) nc = 1184;
        if (t_counts.l1) update_counts<true><<<(unsigned)nc, kThreads, 0, s>>>(counts, c0, c1, t_counts);
        else update_counts<false><<<(unsigned)nc, kThreads, 0, s>>>(counts, c0, c1, t_counts);
        if (launches) *launches += 3;
        return cudaGetLastError();
    }
    if (tr) update_elems<true><<<(unsigned)nb, kThreads, 0, s>>>(sums, counts, cen, c0, c1, d, shift, t_sums, t_cen);
    else update_elems<false><<<(unsigned)nb, kThreads, 0, s>>>(sums, counts, cen, c0, c1, d, shift, t_sums, t_cen);
    int64_t nc = (c1 - c0 + kThreads - 1) / kThreads;
    if (nc > 1184) nc = 1184;
    if (t_counts.l1) update_counts<true><<<(unsigned)nc, kThreads, 0, s>>>(counts, c0, c1, t_counts);
    else update_counts<false><<<(unsigned)nc, kThreads, 0, s>>>(counts, c0, c1, t_counts);
    if (launches) *launches += 2;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
