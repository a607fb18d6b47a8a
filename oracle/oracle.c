/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, sequential CPU implementation of what one offloaded parallel loop of
 * Komoda et al. (ICPP'13, /root/reference/PAPER.md, cited as "L<line> §<section>")
 * computes, over ONE host copy of every array. Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library. The product
 * (paper_conf_icpp_komodamnm13_b200/) never includes, links or calls it, and this file
 * includes nothing from the product tree.
 *
 * Build: gcc -O2 -ffp-contract=off -fopenmp (no FMA contraction: every fused multiply-add
 * below is an explicit fmaf). The OpenMP pragmas only split independent outer iterations
 * (rows / points / output rows); no sum is reordered, so results are bitwise independent of
 * the thread count (tested).
 *
 * Parity status per function: see the "pin:" line of each; none is "parity unpinned".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

static int nthr(int n) { return n > 0 ? n : omp_get_max_threads(); }

/* ------------------------------------------------------------------------------------ */
/* Task mapping — L108 §IV.B.2 "the tasks in the parallel loop are equally divided among
 * the GPUs"; remainder reading G6: chunk g = [lo + floor(g*n/P), lo + floor((g+1)*n/P)).
 * pin: tests/test_oracle_host.py — brute-force coverage/contiguity/balance for n<=64, P<=9. */
void orc_partition(int64_t lo, int64_t hi, int P, int g, int64_t* a, int64_t* b) {
    __int128 n = hi - lo;
    *a = lo + (int64_t)((n * g) / P);
    *b = lo + (int64_t)((n * (g + 1)) / P);
}

/* Partition that owns iteration i (first g with a_g <= i < b_g), -1 if outside [lo, hi). */
int orc_owner(int64_t lo, int64_t hi, int P, int64_t i) {
    for (int g = 0; g < P; ++g) {
        int64_t a, b;
        orc_partition(lo, hi, P, g, &a, &b);
        if (i >= a && i < b) return g;
    }
    return -1;
}

/* localaccess window of ONE iteration — L87 §III.C: "the i-th iteration of the loop use the
 * array elements whose indices are from the range stride*i - left to stride*(i+1) - 1 + right".
 * Returned half-open [lo, hi) (inclusive upper bound + 1), not clipped.
 * pin: tests — union over a chunk equals the closed form; C1 worked example. */
void orc_window_iter(int64_t stride, int64_t left, int64_t right, int64_t i, int64_t* lo, int64_t* hi) {
    *lo = stride * i - left;
    *hi = stride * (i + 1) - 1 + right + 1;
}

/* ------------------------------------------------------------------------------------ */
/* Dirty bits — L133 §IV.D.1 "turn on the dirty bits for every writes accesses to the
 * replicated arrays"; granularity reading G8: 1 bit per element, bit b of uint32 word w is
 * element 32w+b. */
static inline void set_bit(uint32_t* bm, int64_t e) { bm[e >> 5] |= 1u << (e & 31); }
static inline int get_bit(const uint32_t* bm, int64_t e) { return (bm[e >> 5] >> (e & 31)) & 1u; }

/* Second-level bits — L135 §IV.D.1: the dirty-bit array "is subdivided into chunks whose sizes
 * are constant. Each chunk also maintains single bit" (polarity reading G10: 1 = the chunk
 * holds >= 1 dirty element). chunk_elems = dirty_chunk_bytes / elem_size (reading G9).
 * pin: tests — Jacobi closed form (chunks overlapping the partition's rows) + brute force. */
void orc_l2_bits(const uint32_t* l1, int64_t extent, int64_t chunk_elems, uint32_t* l2) {
    int64_t nchunks = (extent + chunk_elems - 1) / chunk_elems;
    memset(l2, 0, sizeof(uint32_t) * (size_t)((nchunks + 31) / 32));
    for (int64_t e = 0; e < extent; ++e)
        if (get_bit(l1, e)) set_bit(l2, e / chunk_elems);
}

/* Canonical packed send buffer (north star (4); format fixed in SURVEY §8.3):
 *   uint64 n_runs, uint64 n_elems, int64 run_start[n_runs], int64 run_end[n_runs] (exclusive),
 *   payload: elem_size * n_elems bytes, the values of every dirty element, runs in ascending order.
 * Runs are the maximal runs of 1-bits of the L1 bitmap. Returns the byte size; writes only if
 * out != NULL. pin: tests — naive maximal-run search (Python) on random bitmaps; Jacobi closed
 * form (one run per row [rN+1, rN+N-1)); C1 worked example 131,080 B. */
int64_t orc_pack(const uint32_t* l1, int64_t extent, const void* values, int64_t esize, uint8_t* out) {
    int64_t n_runs = 0, n_elems = 0;
    for (int64_t e = 0; e < extent; ++e) {
        int b = get_bit(l1, e);
        if (b) { n_elems++; if (e == 0 || !get_bit(l1, e - 1)) n_runs++; }
    }
    int64_t bytes = 16 + 16 * n_runs + esize * n_elems;
    if (!out) return bytes;
    uint64_t* hdr = (uint64_t*)out;
    hdr[0] = (uint64_t)n_runs; hdr[1] = (uint64_t)n_elems;
    int64_t* rs = (int64_t*)(out + 16);
    int64_t* re = rs + n_runs;
    uint8_t* pay = out + 16 + 16 * n_runs;
    int64_t r = 0, p = 0;
    for (int64_t e = 0; e < extent; ++e) {
        if (!get_bit(l1, e)) continue;
        if (e == 0 || !get_bit(l1, e - 1)) rs[r] = e;
        if (e == extent - 1 || !get_bit(l1, e + 1)) { re[r] = e + 1; r++; }
        memcpy(pay + p * esize, (const uint8_t*)values + e * esize, (size_t)esize);
        p++;
    }
    return bytes;
}

/* Receiver side of the packed buffer: write each run's payload at the same global indices. */
void orc_unpack(const uint8_t* packed, void* values, int64_t esize) {
    const uint64_t* hdr = (const uint64_t*)packed;
    int64_t n_runs = (int64_t)hdr[0];
    const int64_t* rs = (const int64_t*)(packed + 16);
    const int64_t* re = rs + n_runs;
    const uint8_t* pay = packed + 16 + 16 * n_runs;
    int64_t p = 0;
    for (int64_t r = 0; r < n_runs; ++r)
        for (int64_t e = rs[r]; e < re[r]; ++e, ++p)
            memcpy((uint8_t*)values + e * esize, pay + p * esize, (size_t)esize);
}

/* ------------------------------------------------------------------------------------ */
/* 2-D 5-point Jacobi sweep (configs C1, C2, C5; the paper has no stencil — the loop body is
 * the workload's, reading W1). Loop rows i in [1, N-1) (the partitioned outer loop, L108),
 * columns j in [1, N-1):
 *     dst[i][j] = 0.25f * ((src[i-1][j] + src[i+1][j]) + (src[i][j-1] + src[i][j+1]))
 * Boundary rows/columns are never written (Dirichlet). If bitmaps != NULL (P bitmaps of
 * ceil(N*N/32) words each, caller-zeroed), every write by an iteration of partition g sets bit
 * i*N+j of bitmaps[g] (L133). pin: tests — constant and integer-linear fixed points, transpose
 * and reflection equivariance, dyadic tiny grids vs exact rationals, partition invariance. */
void orc_jacobi_sweep(const float* src, float* dst, int64_t N, int P, uint32_t* bitmaps, int nthreads) {
    int64_t nwords = (N * N + 31) / 32;
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t i = 1; i < N - 1; ++i) {
        for (int64_t j = 1; j < N - 1; ++j) {
            float ns = src[(i - 1) * N + j] + src[(i + 1) * N + j];
            float we = src[i * N + j - 1] + src[i * N + j + 1];
            dst[i * N + j] = 0.25f * (ns + we);
        }
    }
    if (bitmaps) {
        for (int64_t i = 1; i < N - 1; ++i) {
            int g = orc_owner(1, N - 1, P, i);
            for (int64_t j = 1; j < N - 1; ++j) set_bit(bitmaps + (int64_t)g * nwords, i * N + j);
        }
    }
}

/* The same sweep on a rows x cols array (rows [1, rows-1), columns [1, cols-1)); used to time
 * the oracle on full-width bands of the C2 field (bench.py cpu_baseline). */
void orc_jacobi_sweep_rect(const float* src, float* dst, int64_t rows, int64_t cols, int nthreads) {
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t i = 1; i < rows - 1; ++i) {
        for (int64_t j = 1; j < cols - 1; ++j) {
            float ns = src[(i - 1) * cols + j] + src[(i + 1) * cols + j];
            float we = src[i * cols + j - 1] + src[i * cols + j + 1];
            dst[i * cols + j] = 0.25f * (ns + we);
        }
    }
}

/* S sweeps alternating A -> B -> A ...: sweep s reads A if s is even (else B) and writes the
 * other. Result in A for even S (reading W1). B must hold a copy of A on entry. */
void orc_jacobi_run(float* A, float* B, int64_t N, int S, int nthreads) {
    for (int s = 0; s < S; ++s) {
        if (s % 2 == 0) orc_jacobi_sweep(A, B, N, 1, NULL, nthreads);
        else orc_jacobi_sweep(B, A, N, 1, NULL, nthreads);
    }
}

/* Sparse-write test loop (T9, exercises L2-chunk skipping, L135): rows i in [0, N); iteration
 * i writes only if i % period == 0:   out[i][j] = in[i][j] + 1.0f  for all j in [0, N). */
void orc_sparse_rows(const float* in, float* out, int64_t N, int64_t period, int P, uint32_t* bitmaps) {
    int64_t nwords = (N * N + 31) / 32;
    for (int64_t i = 0; i < N; ++i) {
        if (i % period != 0) continue;
        int g = orc_owner(0, N, P, i);
        for (int64_t j = 0; j < N; ++j) {
            out[i * N + j] = in[i * N + j] + 1.0f;
            if (bitmaps) set_bit(bitmaps + (int64_t)g * nwords, i * N + j);
        }
    }
}

/* Masked-write test loop (exercises the dirty-bit compaction of L133-135 with arbitrary bit
 * patterns): iterations e in [0, n); iteration e writes only if mask[e] != 0:
 *   out[e] = in[e] + 1.0f.   Bit e of partition orc_owner(0, n, P, e)'s bitmap is set per write.
 * pin: tests — brute-force Python loop on small n, bitmaps = mask bits split by partition. */
void orc_masked_write(const float* in, const uint8_t* mask, float* out, int64_t n, int P, uint32_t* bitmaps) {
    int64_t nwords = (n + 31) / 32;
    for (int64_t e = 0; e < n; ++e) {
        if (!mask[e]) continue;
        out[e] = in[e] + 1.0f;
        if (bitmaps) set_bit(bitmaps + (int64_t)orc_owner(0, n, P, e) * nwords, e);
    }
}

/* ------------------------------------------------------------------------------------ */
/* Dense matmul (config C3): R[i][j] = sum_{k=0}^{K-1} (double)A[i][k] * (double)B[k][j],
 * k ascending, fp64. A, B are bf16 bit patterns (row-major [M][K], [K][N]); bf16 -> fp64 is
 * exact and so is each product (8+8 significand bits). Computes only the listed rows.
 * (Loop order k-outer/j-inner keeps each R[i][j] an ascending-k sum.)
 * pin: tests — identity, rank-1 products and small-integer inputs against Python integers. */
static inline double bf16d(uint16_t h) {
    uint32_t b = (uint32_t)h << 16; float f; memcpy(&f, &b, 4); return (double)f;
}
void orc_gemm_rows_f64(const uint16_t* A, const uint16_t* B, int64_t M, int64_t N, int64_t K,
                       const int64_t* rows, int64_t nrows, double* out, int nthreads) {
    (void)M;
    #pragma omp parallel for schedule(dynamic) num_threads(nthr(nthreads))
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t i = rows[r];
        double* acc = out + r * N;
        for (int64_t j = 0; j < N; ++j) acc[j] = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            double a = bf16d(A[i * K + k]);
            const uint16_t* brow = B + k * N;
            for (int64_t j = 0; j < N; ++j) acc[j] += a * bf16d(brow[j]);
        }
    }
}

/* ------------------------------------------------------------------------------------ */
/* k-means (config C4; KMEANS is the paper's Rodinia workload, Table II; the loop
 * semantics below are readings stated in SURVEY §8.3 and DESIGN.md).
 * Assignment loop over points p (partitioned, L108): best = 0, bestd = +inf; for c = 0..k-1:
 * acc = 0.0f; for j = 0..d-1: diff = x[p][j] - cen[c][j] (fp32 RN); acc = fmaf(diff, diff, acc);
 * if (acc < bestd) {bestd = acc; best = c}. Ties -> lowest index.
 * pin: tests — lattice clusters recover labels; integer brute force; tie and empty-cluster cases. */
void orc_kmeans_assign(const float* x, int64_t n, int d, int k, const float* cen, int32_t* member,
                       int nthreads) {
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t p = 0; p < n; ++p) {
        int best = 0;
        float bestd = INFINITY;
        for (int c = 0; c < k; ++c) {
            float acc = 0.0f;
            for (int j = 0; j < d; ++j) {
                float diff = x[p * d + j] - cen[(int64_t)c * d + j];
                acc = fmaf(diff, diff, acc);
            }
            if (acc < bestd) { bestd = acc; best = c; }
        }
        member[p] = best;
    }
}

/* reductiontoarray (L75-77 §III.B, L89-91 §III.C): sum[member[p]][j] += (double)x[p][j];
 * cnt[member[p]] += 1 — sequential in p. Then the update loop over clusters:
 * cen[c][j] = (float)(sum[c][j] / (double)cnt[c]) if cnt[c] > 0, else unchanged.
 * Writes the sums/counts it used (sum: k*d doubles, cnt: k int64) if non-NULL. */
void orc_kmeans_update(const float* x, int64_t n, int d, int k, const int32_t* member, float* cen,
                       double* sum_out, int64_t* cnt_out) {
    double* sum = (double*)calloc((size_t)k * d, sizeof(double));
    int64_t* cnt = (int64_t*)calloc((size_t)k, sizeof(int64_t));
    for (int64_t p = 0; p < n; ++p) {
        int m = member[p];
        for (int j = 0; j < d; ++j) sum[(int64_t)m * d + j] += (double)x[p * d + j];
        cnt[m] += 1;
    }
    for (int c = 0; c < k; ++c)
        if (cnt[c] > 0)
            for (int j = 0; j < d; ++j) cen[(int64_t)c * d + j] = (float)(sum[(int64_t)c * d + j] / (double)cnt[c]);
    if (sum_out) memcpy(sum_out, sum, sizeof(double) * (size_t)k * d);
    if (cnt_out) memcpy(cnt_out, cnt, sizeof(int64_t) * (size_t)k);
    free(sum); free(cnt);
}

/* Full run: cen[c] = x[c] for c < k, then `iters` x (assignment, update).
 * Outputs member from the last assignment and cen after the last update. */
void orc_kmeans_run(const float* x, int64_t n, int d, int k, int iters, float* cen, int32_t* member,
                    int nthreads) {
    for (int c = 0; c < k; ++c) memcpy(cen + (int64_t)c * d, x + (int64_t)c * d, sizeof(float) * d);
    for (int it = 0; it < iters; ++it) {
        orc_kmeans_assign(x, n, d, k, cen, member, nthreads);
        orc_kmeans_update(x, n, d, k, member, cen, NULL, NULL);
    }
}

/* ------------------------------------------------------------------------------------ */
/* Irregular writes to a distributed array (L137 §IV.D.2; §8 row f1; the BFS class of L173):
 * loop i in [lo, hi): dst[idx[i]] = src[i], sequential. If P > 0, miss[g] = the number of writes by
 * partition g's iterations whose index lies outside g's declared write window [a_g, b_g) (stride 1,
 * the window of iterations [a_g, b_g) of the same loop bounds). pin: tests — identity and reversal
 * permutations, scatter-then-inverse-scatter identity, brute-force miss counts. */
void orc_scatter(const float* src, const int32_t* idx, float* dst, int64_t lo, int64_t hi, int P, int64_t* miss) {
    for (int64_t i = lo; i < hi; ++i) dst[idx[i]] = src[i];
    if (miss && P > 0) {
        for (int g = 0; g < P; ++g) {
            int64_t a, b;
            orc_partition(lo, hi, P, g, &a, &b);
            miss[g] = 0;
            for (int64_t i = a; i < b; ++i)
                if (idx[i] < a || idx[i] >= b) miss[g]++;
        }
    }
}

/* ------------------------------------------------------------------------------------ */
/* 3-D 7-point Jacobi sweep (§8 row f2; multi-dimensional stencils, L256; reading in DESIGN.md):
 * for i in [1,n0-1) (partitioned), j in [1,n1-1), k in [1,n2-1):
 *   dst = ((((u + d) + (n + s)) + ((w + e) + (c + c))) * 0.125f
 * u/d = src[i-1/i+1][j][k], n/s = src[i][j-1/j+1][k], w/e = src[i][j][k-1/k+1], c = src[i][j][k].
 * Bitmaps as for the 2-D sweep (plane i belongs to partition orc_owner(1, n0-1, P, i)).
 * pin: tests — constant and integer-linear fixed points, axis reflections, dyadic exact rationals. */
void orc_jacobi3d_sweep(const float* src, float* dst, int64_t n0, int64_t n1, int64_t n2, int P, uint32_t* bitmaps,
                        int nthreads) {
    int64_t E = n0 * n1 * n2, nwords = (E + 31) / 32, pl = n1 * n2;
    #pragma omp parallel for schedule(static) num_threads(nthr(nthreads))
    for (int64_t i = 1; i < n0 - 1; ++i)
        for (int64_t j = 1; j < n1 - 1; ++j)
            for (int64_t k = 1; k < n2 - 1; ++k) {
                int64_t x = i * pl + j * n2 + k;
                float ud = src[x - pl] + src[x + pl];
                float ns = src[x - n2] + src[x + n2];
                float we = src[x - 1] + src[x + 1];
                float cc = src[x] + src[x];
                dst[x] = ((ud + ns) + (we + cc)) * 0.125f;
            }
    if (bitmaps)
        for (int64_t i = 1; i < n0 - 1; ++i) {
            int g = orc_owner(1, n0 - 1, P, i);
            for (int64_t j = 1; j < n1 - 1; ++j)
                for (int64_t k = 1; k < n2 - 1; ++k) set_bit(bitmaps + (int64_t)g * nwords, i * pl + j * n2 + k);
        }
}

void orc_jacobi3d_run(float* A, float* B, int64_t n0, int64_t n1, int64_t n2, int S, int nthreads) {
    for (int s = 0; s < S; ++s) {
        if (s % 2 == 0) orc_jacobi3d_sweep(A, B, n0, n1, n2, 1, NULL, nthreads);
        else orc_jacobi3d_sweep(B, A, n0, n1, n2, 1, NULL, nthreads);
    }
}
