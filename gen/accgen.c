/*
 * accgen — seeded, counter-based synthetic input generators.
 *
 * This module is shared by the oracle tests, the GPU parity tests and bench.py.
 * It holds NONE of the method's arithmetic (no stencil, no GEMM, no k-means,
 * no partitioning, no coherence logic): only the SplitMix64 counter generator
 * and the value recipes of the synthetic workloads, stated in DESIGN.md §Inputs.
 *
 *   u(seed, i) = mix(seed * 0x9E3779B97F4A7C15 + (i + 1) * 0xD1B54A32D192ED03)  (mod 2^64)
 *   mix(x): x ^= x >> 30; x *= 0xBF58476D1CE4E5B9; x ^= x >> 27;
 *           x *= 0x94D049BB133111EB; x ^= x >> 31
 *
 * Every element depends only on (seed, index), so any row range can be produced
 * independently (one rank can generate just its window) and the result never
 * depends on the thread count.
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC (see Makefile).
 */
#include <stdint.h>
#include <string.h>
#include <omp.h>

#define GOLD 0x9E3779B97F4A7C15ULL
#define STEP 0xD1B54A32D192ED03ULL

static inline uint64_t mix64(uint64_t x) {
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ULL;
    x ^= x >> 27; x *= 0x94D049BB133111EBULL;
    x ^= x >> 31;
    return x;
}

uint64_t accgen_u(uint64_t seed, uint64_t i) { return mix64(seed * GOLD + (i + 1) * STEP); }

static inline float unit24(uint64_t u) { return (float)(u >> 40) * (1.0f / 16777216.0f); }

/* nthreads <= 0: all OpenMP threads. Results never depend on the thread count. */
static int nthr(int n) { return n > 0 ? n : omp_get_max_threads(); }

void accgen_u_fill(uint64_t seed, uint64_t i0, int64_t n, uint64_t* out) {
    for (int64_t k = 0; k < n; ++k) out[k] = accgen_u(seed, i0 + (uint64_t)k);
}

/* Jacobi field (configs C1/C2/C5): N x N fp32, row-major.
 * Row 0 = 1.0 (including its corners); rows N-1 and columns 0, N-1 = 0 elsewhere;
 * interior (i,j) = (u(seed, i*N+j) >> 40) * 2^-24, uniform on [0,1), exact in fp32.
 * Writes rows [r0, r1) to out[(r - r0) * N + j]. */
void accgen_jacobi_rows(uint64_t seed, int64_t N, int64_t r0, int64_t r1, float* out, int nthreads) {
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t r = r0; r < r1; ++r) {
        float* row = out + (r - r0) * N;
        if (r == 0) { for (int64_t j = 0; j < N; ++j) row[j] = 1.0f; continue; }
        if (r == N - 1) { for (int64_t j = 0; j < N; ++j) row[j] = 0.0f; continue; }
        row[0] = 0.0f; row[N - 1] = 0.0f;
        for (int64_t j = 1; j < N - 1; ++j) row[j] = unit24(accgen_u(seed, (uint64_t)(r * N + j)));
    }
}

static inline uint16_t f32_to_bf16_rne(float f) {
    uint32_t b; memcpy(&b, &f, 4);
    uint32_t rounding = ((b >> 16) & 1u) + 0x7FFFu;
    return (uint16_t)((b + rounding) >> 16);
}

/* bf16 matrix [rows][cols], rows [r0, r1) written to out[(r-r0)*cols + c].
 * kind 0: integers in {-2..2}: u % 5 - 2 (exact in bf16).
 * kind 1: uniform (0,1]: ((u >> 40) + 1) * 2^-24 rounded to nearest-even bf16.
 * kind 2: signed uniform [-1,1): 2*(u>>40)*2^-24 - 1 rounded to nearest-even bf16. */
void accgen_bf16_matrix(uint64_t seed, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                        int kind, uint16_t* out, int nthreads) {
    (void)rows;
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t r = r0; r < r1; ++r) {
        uint16_t* row = out + (r - r0) * cols;
        for (int64_t c = 0; c < cols; ++c) {
            uint64_t u = accgen_u(seed, (uint64_t)(r * cols + c));
            float v;
            if (kind == 0) v = (float)((int)(u % 5) - 2);
            else if (kind == 1) v = (float)((u >> 40) + 1) * (1.0f / 16777216.0f);
            else v = 2.0f * (float)(u >> 40) * (1.0f / 16777216.0f) - 1.0f;
            row[c] = f32_to_bf16_rne(v);
        }
    }
}

/* k-means centres [k][d]. mode 0 (lattice, C4 closed form): coordinate -64 + 16*(u % 8).
 * mode 1 (overlapping, C4 parity set): coordinate -8 + (u % 16).
 * Centre c, coordinate j, attempt a draws u(seed, c*d + j + a*2^40); a centre equal to an
 * earlier centre in all d coordinates is redrawn with the next attempt. */
void accgen_kmeans_centres(uint64_t seed, int k, int d, int mode, float* centres) {
    for (int c = 0; c < k; ++c) {
        for (uint64_t a = 0;; ++a) {
            for (int j = 0; j < d; ++j) {
                uint64_t u = accgen_u(seed, (uint64_t)c * (uint64_t)d + (uint64_t)j + (a << 40));
                centres[(int64_t)c * d + j] = mode == 0 ? (float)(-64 + 16 * (int)(u % 8))
                                                        : (float)(-8 + (int)(u % 16));
            }
            int dup = 0;
            for (int c2 = 0; c2 < c && !dup; ++c2)
                dup = memcmp(centres + (int64_t)c2 * d, centres + (int64_t)c * d, sizeof(float) * d) == 0;
            if (!dup) break;
        }
    }
}

/* k-means points [n][d], points [p0, p1) written to out[(p-p0)*d + j] (labels optional).
 * label(p) = p for p < k, else u(seed+1, p) % k.
 * noise(p,j): mode 0: ((u(seed+2, p*d+j) % 257) - 128) / 256; mode 1: ((u % 1025) - 512) / 256.
 * x = centre[label][j] + noise: both on the 2^-8 grid with |x| < 128, so the sum is exact. */
void accgen_kmeans_points(uint64_t seed, int64_t n, int d, int k, int mode, const float* centres,
                          int64_t p0, int64_t p1, float* out, int32_t* labels, int nthreads) {
    (void)n;
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t p = p0; p < p1; ++p) {
        int lab = p < k ? (int)p : (int)(accgen_u(seed + 1, (uint64_t)p) % (uint64_t)k);
        if (labels) labels[p - p0] = lab;
        for (int j = 0; j < d; ++j) {
            uint64_t u = accgen_u(seed + 2, (uint64_t)p * (uint64_t)d + (uint64_t)j);
            int q = mode == 0 ? (int)(u % 257) - 128 : (int)(u % 1025) - 512;
            out[(p - p0) * d + j] = centres[(int64_t)lab * d + j] + (float)q * (1.0f / 256.0f);
        }
    }
}

/* Random permutation of [0, n) (Fisher-Yates, swap i with u(seed, i) % (i + 1), i = n-1 .. 1):
 * the index array of the irregular-write (scatter) workload. */
void accgen_permutation(uint64_t seed, int64_t n, int32_t* out) {
    for (int64_t i = 0; i < n; ++i) out[i] = (int32_t)i;
    for (int64_t i = n - 1; i > 0; --i) {
        int64_t j = (int64_t)(accgen_u(seed, (uint64_t)i) % (uint64_t)(i + 1));
        int32_t t = out[i]; out[i] = out[j]; out[j] = t;
    }
}

/* 3-D Jacobi field (row f2): n0 x n1 x n2 fp32, planes [i0, i1) written to out. Plane 0 = 1.0; the
 * other boundary faces 0; interior (i,j,k) = (u(seed, (i*n1+j)*n2+k) >> 40) * 2^-24. */
void accgen_field3d(uint64_t seed, int64_t n0, int64_t n1, int64_t n2, int64_t i0, int64_t i1, float* out,
                    int nthreads) {
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t i = i0; i < i1; ++i)
        for (int64_t j = 0; j < n1; ++j)
            for (int64_t k = 0; k < n2; ++k) {
                const int64_t x = (i * n1 + j) * n2 + k;
                float v;
                if (i == 0) v = 1.0f;
                else if (i == n0 - 1 || j == 0 || j == n1 - 1 || k == 0 || k == n2 - 1) v = 0.0f;
                else v = unit24(accgen_u(seed, (uint64_t)x));
                out[x - i0 * n1 * n2] = v;
            }
}
