// Loop body: 2-D 5-point Jacobi sweep on one partition's row chunk (configs C1, C2, C5).
//
//   dst[i][j] = 0.25f * ((src[i-1][j] + src[i+1][j]) + (src[i][j-1] + src[i][j+1]))
//   for i in [r0, r1) (this partition's chunk of the divided outer loop, L108 §IV.B.2),
//       j in [c0, c1); boundary rows/columns are never stored (reading W1/W2).
//
// HBM-bound: 4 B read + 4 B written per point (8 B algorithmic traffic), 4 flop. Design
// (B200): each warp owns a 128-column strip (32 lanes x float4) and marches down a segment of
// rows, keeping rows i-1, i, i+1 in registers, so every input element is read from HBM once
// (plus 2 halo rows per segment); horizontal neighbours come from warp shuffles, the two strip
// edges from one scalar load each. kUnroll rows are loaded before any is consumed (4 x 16 B in
// flight per lane) to cover HBM latency. Stores are full 128-bit and coalesced except on the
// two boundary columns. Arithmetic uses explicit round-to-nearest adds/multiplies in the
// parenthesisation above, so results are bit-identical to the oracle for any partition count.
// The optional fused epilogue (TRACK) sets the two-level dirty bits of every written element
// (L133-135) with warp-aggregated atomics (track.cuh).
#include <cstdlib>

#include "kernels.h"
#include "track.cuh"

namespace accmg {
namespace k {
namespace {

constexpr int kWarps = 8;          // warps per CTA (8 adjacent column strips)
constexpr int kRowsPerSeg = 128;   // rows one warp marches through (2 halo rows re-read per segment)
constexpr int kUnrollPlain = 4;    // rows loaded ahead (untracked body: 0.97 of copy peak)
constexpr int kUnrollTrack = 4;    // tracked body: same pipeline, tracking done after the row loop

template <int VEC>
struct Row {
    float v[VEC];
};

template <int VEC>
__device__ __forceinline__ Row<VEC> ldrow(const float* __restrict__ p, bool ok) {
    Row<VEC> r;
    if constexpr (VEC == 4) {
        float4 f = ok ? __ldg(reinterpret_cast<const float4*>(p)) : make_float4(0.f, 0.f, 0.f, 0.f);
        r.v[0] = f.x; r.v[1] = f.y; r.v[2] = f.z; r.v[3] = f.w;
    } else {
        r.v[0] = ok ? __ldg(p) : 0.f;
    }
    return r;
}

// ((n + s) + (w + e)) * 0.25f with explicit RN operations (no contraction, fixed order)
__device__ __forceinline__ float st5(float n, float s, float w, float e) {
    return __fmul_rn(__fadd_rn(__fadd_rn(n, s), __fadd_rn(w, e)), 0.25f);
}

template <int VEC, bool TRACK, int kUnroll = TRACK ? kUnrollTrack : kUnrollPlain>
__global__ void __launch_bounds__(kWarps * 32, 4)
jacobi_rows(const float* __restrict__ src, float* __restrict__ dst, int64_t cols, int64_t r0, int64_t r1,
            int64_t c0, int64_t c1, int64_t cbase, Track t, const HaloPush push) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t cw = cbase + ((int64_t)blockIdx.x * kWarps + warp) * (32 * VEC);  // warp's first column
    if (cw >= c1) return;                                                           // warp-uniform
    const int64_t c = cw + VEC * lane;
    const int64_t rs = r0 + (int64_t)blockIdx.y * kRowsPerSeg;
    const int64_t re = rs + kRowsPerSeg < r1 ? rs + kRowsPerSeg : r1;
    const bool in_cols = c + VEC <= cols;
    unsigned nib = 0;
#pragma unroll
    for (int k = 0; k < VEC; ++k) nib |= (c + k >= c0 && c + k < c1) ? (1u << k) : 0u;
    const bool full = nib == (1u << VEC) - 1u;
    const bool hw_ok = lane == 0 && c >= 1;
    const bool he_ok = lane == 31 && c + VEC < cols;

    Row<VEC> rb[kUnroll + 2];  // rb[0] = row i-1, rb[1] = row i, rb[2..] = rows i+1 .. i+kUnroll
    rb[0] = ldrow<VEC>(src + (rs - 1) * cols + c, in_cols);
    rb[1] = ldrow<VEC>(src + rs * cols + c, in_cols);
    dev::WarpTracker<VEC> trk;
    if constexpr (TRACK) trk.init(nib);
    for (int64_t i = rs; i < re; i += kUnroll) {
        float hw[kUnroll], he[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            const int64_t r = i + u;
            const bool ok = r < re;  // warp-uniform
            rb[u + 2] = ldrow<VEC>(src + (r + 1) * cols + c, ok && in_cols);
            hw[u] = (ok && hw_ok) ? __ldg(src + r * cols + c - 1) : 0.f;
            he[u] = (ok && he_ok) ? __ldg(src + r * cols + c + VEC) : 0.f;
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            const int64_t r = i + u;
            if (r >= re) break;
            const Row<VEC>& up = rb[u];
            const Row<VEC>& ce = rb[u + 1];
            const Row<VEC>& dn = rb[u + 2];
            float w = __shfl_up_sync(dev::kFull, ce.v[VEC - 1], 1);
            float e = __shfl_down_sync(dev::kFull, ce.v[0], 1);
            if (lane == 0) w = hw[u];
            if (lane == 31) e = he[u];
            float o[VEC];
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                const float west = k == 0 ? w : ce.v[k > 0 ? k - 1 : 0];
                const float east = k == VEC - 1 ? e : ce.v[k < VEC - 1 ? k + 1 : 0];
                o[k] = st5(up.v[k], dn.v[k], west, east);
            }
            float* q = dst + r * cols + c;
            if constexpr (VEC == 4) {
                if (full) {
                    *reinterpret_cast<float4*>(q) = make_float4(o[0], o[1], o[2], o[3]);
                } else {
#pragma unroll
                    for (int k = 0; k < VEC; ++k)
                        if (nib & (1u << k)) q[k] = o[k];
                }
            } else {
                if (nib) q[0] = o[0];
            }
            if (push.n) {  // predicted readers' copies (rare rows; static indices)
#pragma unroll
                for (int pi = 0; pi < kMaxPush; ++pi) {
                    if (pi >= push.n || r < push.lo[pi] || r >= push.hi[pi]) continue;  // warp-uniform
                    float* pq = push.dst[pi] + r * cols + c;
#pragma unroll
                    for (int k = 0; k < VEC; ++k)
                        if (nib & (1u << k)) pq[k] = o[k];
                }
            }
        }
        rb[0] = rb[kUnroll];
        rb[1] = rb[kUnroll + 1];
    }
    // fused dirty tracking of every element this warp wrote (rows [rs, re) of its strip)
    if constexpr (TRACK) trk.mark_rows(t.l1, t.l2, t.l2_shift, rs, re, cols, cw);
}

template <int VEC>
cudaError_t launch_rows(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                        int64_t c0, int64_t c1, Track t, const HaloPush& push, cudaStream_t s) {
    (void)rows;
    const int64_t span = 32 * VEC * kWarps;
    const int64_t cbase = (c0 / (32 * VEC)) * (32 * VEC);
    dim3 grid((unsigned)((c1 - cbase + span - 1) / span), (unsigned)((r1 - r0 + kRowsPerSeg - 1) / kRowsPerSeg));
    if (t.l1)
        jacobi_rows<VEC, true><<<grid, kWarps * 32, 0, s>>>(src, dst, cols, r0, r1, c0, c1, cbase, t, push);
    else
        jacobi_rows<VEC, false><<<grid, kWarps * 32, 0, s>>>(src, dst, cols, r0, r1, c0, c1, cbase, t, push);
    return cudaGetLastError();
}

// Test body (T9): rows i in [r0, r1) with i % period == 0 get out[i][:] = in[i][:] + 1.0f.
template <bool TRACK>
__global__ void __launch_bounds__(256)
sparse_rows_kernel(const float* __restrict__ in, float* __restrict__ out, int64_t cols, int64_t first,
                   int64_t r1, int64_t period, Track t) {
    const int64_t c = (int64_t)blockIdx.x * 256 + threadIdx.x;
    const int64_t cw = c - (threadIdx.x & 31);
    int64_t l2c = -1;
    for (int64_t i = first + (int64_t)blockIdx.y * period; i < r1; i += (int64_t)gridDim.y * period) {
        const bool ok = c < cols;
        if (ok) out[i * cols + c] = __fadd_rn(in[i * cols + c], 1.0f);
        if constexpr (TRACK) {
            if (cw < cols) dev::track_warp<1>(t.l1, t.l2, t.l2_shift, i * cols + cw, ok ? 1u : 0u, l2c);
        }
    }
}

template <bool TRACK>
__global__ void __launch_bounds__(256)
masked_write_kernel(const float* __restrict__ in, const uint8_t* __restrict__ mask, float* __restrict__ out, int64_t e0,
                    int64_t e1, Track t) {
    const int lane = threadIdx.x & 31;
    int64_t l2c = -1;
    for (int64_t base = e0 + ((int64_t)blockIdx.x * 256 + threadIdx.x - lane); base < e1;
         base += (int64_t)gridDim.x * 256) {
        const int64_t e = base + lane;
        const bool w = e < e1 && mask[e] != 0;
        if (w) out[e] = __fadd_rn(in[e], 1.0f);
        if constexpr (TRACK) dev::track_warp<1>(t.l1, t.l2, t.l2_shift, base, w ? 1u : 0u, l2c);
    }
}

}  // namespace

cudaError_t jacobi2d(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                     int64_t c0, int64_t c1, int64_t src_lo, int64_t src_hi, Track t, int impl, cudaStream_t s,
                     int64_t* launches, const HaloPush& push) {
    if (r1 <= r0 || c1 <= c0) return cudaSuccess;
    // impl 0: TMA-staged tiles (measured faster, profiles/r01/jacobi_impl.log) where the shape
    // allows; shapes the TMA body does not take (and impl 1) run the register row-marching kernel
    if (impl == 0) {
        cudaError_t e = jacobi2d_tma(src, dst, rows, cols, r0, r1, c0, c1, src_lo, src_hi, t, s, launches, push);
        if (e != cudaErrorNotSupported) return e;  // shapes the TMA variant does not take fall through
    }
    uintptr_t align = reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst);
    for (int i = 0; i < push.n; ++i) align |= reinterpret_cast<uintptr_t>(push.dst[i]);  // pushed rows are stored alike
    const bool vec4 = (cols % 4 == 0) && align % 16 == 0;
    cudaError_t e = vec4 ? launch_rows<4>(src, dst, rows, cols, r0, r1, c0, c1, t, push, s)
                         : launch_rows<1>(src, dst, rows, cols, r0, r1, c0, c1, t, push, s);
    if (launches) *launches += 1;
    return e;
}

namespace {
__global__ void frame_copy_k(const float* __restrict__ src, float* __restrict__ tmp, int64_t cols, int64_t lo,
                             int64_t hi, int64_t rlo, int64_t rhi, int64_t c0, int64_t c1) {
    for (int64_t r = lo + blockIdx.x; r < hi; r += gridDim.x) {
        const bool whole = r < rlo || r >= rhi;
        for (int64_t c = threadIdx.x; c < cols; c += blockDim.x)
            if (whole || c < c0 || c >= c1) tmp[r * cols + c] = src[r * cols + c];
    }
}
}  // namespace

cudaError_t frame_copy(const float* src, float* tmp, int64_t cols, int64_t lo, int64_t hi, int64_t rlo, int64_t rhi,
                       int64_t c0, int64_t c1, cudaStream_t s, int64_t* launches) {
    if (hi <= lo) return cudaSuccess;
    const int64_t nb = (hi - lo) < 1184 ? (hi - lo) : 1184;
    frame_copy_k<<<(unsigned)nb, 256, 0, s>>>(src, tmp, cols, lo, hi, rlo, rhi, c0, c1);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t sparse_rows(const float* in, float* out, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                        int64_t period, Track t, cudaStream_t s, int64_t* launches) {
    (void)rows;
    const int64_t first = ((r0 + period - 1) / period) * period;
    if (first >= r1) return cudaSuccess;
    const int64_t nsel = (r1 - first + period - 1) / period;
    dim3 grid((unsigned)((cols + 255) / 256), (unsigned)(nsel < 65535 ? nsel : 65535));
    if (t.l1) sparse_rows_kernel<true><<<grid, 256, 0, s>>>(in, out, cols, first, r1, period, t);
    else sparse_rows_kernel<false><<<grid, 256, 0, s>>>(in, out, cols, first, r1, period, t);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

cudaError_t masked_write(const float* in, const uint8_t* mask, float* out, int64_t e0, int64_t e1, Track t,
                         cudaStream_t s, int64_t* launches) {
    if (e1 <= e0) return cudaSuccess;
    int64_t nb = (e1 - e0 + 255) / 256;
    if (nb > 148 * 8) nb = 148 * 8;
    if (t.l1) masked_write_kernel<true><<<(unsigned)nb, 256, 0, s>>>(in, mask, out, e0, e1, t);
    else masked_write_kernel<false><<<(unsigned)nb, 256, 0, s>>>(in, mask, out, e0, e1, t);
    if (launches) *launches += 1;
    return cudaGetLastError();
}

}  // namespace k
}  // namespace accmg
