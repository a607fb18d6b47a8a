"""Pins for the oracle's loop bodies (Jacobi, GEMM, k-means). CPU only.

Every expected value comes from mathematics independent of the oracle's code: fixed points,
symmetry, exact rationals (fractions.Fraction), Python integers, closed forms of the
generated clusters.
"""
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle


# ---- Jacobi (reading W1) ------------------------------------------------------------------
def _sweeps(A, S, P=1):
    A = A.copy()
    B = A.copy()
    oracle.jacobi_run(A, B, S)
    return A if S % 2 == 0 else B


@pytest.mark.parametrize("c", [0.0, 1.0, 0.3, -7.25, 1e30])
def test_constant_field_is_fixed_point(c):
    A = np.full((64, 64), c, dtype=np.float32)
    assert np.array_equal(_sweeps(A, 10), A)


@pytest.mark.parametrize("shape_coef", [(64, 1, 2, 3), (65, -3, 5, 100)])
def test_integer_linear_field_is_fixed_point(shape_coef):
    N, a, b, c = shape_coef
    i, j = np.meshgrid(np.arange(N), np.arange(N), indexing="ij")
    A = (a * i + b * j + c).astype(np.float32)     # harmonic; integers, sums exact in fp32
    assert np.array_equal(_sweeps(A, 10), A)


def test_transpose_and_reflection_equivariance():
    A = gen.jacobi_field(11, 65)
    A[:, 0] = 0.5                                   # make the boundary asymmetric too
    out = _sweeps(A, 10)
    assert np.array_equal(_sweeps(np.ascontiguousarray(A.T), 10), out.T)
    assert np.array_equal(_sweeps(np.ascontiguousarray(A[::-1]), 10), out[::-1])
    assert np.array_equal(_sweeps(np.ascontiguousarray(A[:, ::-1]), 10), out[:, ::-1])


@pytest.mark.parametrize("shape", [(4, 4), (5, 7), (7, 9), (6, 6)])
def test_tiny_dyadic_grids_vs_exact_rationals(shape):
    rng = np.random.default_rng(sum(shape))
    R, C = shape
    N = max(R, C)
    # square array, values k/8 in [0, 2): every intermediate stays exactly representable
    A = (rng.integers(0, 16, (N, N)) / 8.0).astype(np.float32)
    F = [[Fraction(float(v)) for v in row] for row in A]
    for s in range(4):
        G = [row[:] for row in F]
        for i in range(1, N - 1):
            for j in range(1, N - 1):
                G[i][j] = (F[i - 1][j] + F[i + 1][j] + F[i][j - 1] + F[i][j + 1]) / 4
        F = G
        got = _sweeps(A, s + 1)
        exact = np.array([[float(v) for v in row] for row in F])
        assert np.array_equal(got.astype(np.float64), exact)


def test_parenthesisation_reading_w1():
    # ((n + s) + (w + e)) * 0.25 with n = 1, s = 2^-24, w = 2^-24, e = 2^-24:
    # n + s = 1 + 2^-24 rounds to 1 (tie to even); w + e = 2^-23; 1 + 2^-23 is exact.
    # A left-to-right sum (((n + s) + w) + e) gives 1 instead (each 2^-24 is lost).
    t = np.float32(2.0 ** -24)
    A = np.zeros((3, 3), dtype=np.float32)
    A[0, 1], A[2, 1], A[1, 0], A[1, 2] = 1.0, t, t, t
    out = _sweeps(A, 1)
    assert out[1, 1] == np.float32(0.25 * (1.0 + 2.0 ** -23))


def test_thread_count_invariance_and_bitmaps_closed_form():
    N, P = 70, 3
    src = gen.jacobi_field(2, N)
    d1, d2 = src.copy(), src.copy()
    oracle.jacobi_sweep(src, d1, nthreads=1)
    bms = oracle.jacobi_sweep(src, d2, P=P, track=True, nthreads=4)
    assert np.array_equal(d1, d2)
    for g in range(P):
        a, b = oracle.partition(1, N - 1, P, g)
        m = np.zeros((N, N), dtype=bool)
        m[a:b, 1:N - 1] = True
        bits = np.unpackbits(bms[g].view(np.uint8), bitorder="little")[:N * N].astype(bool)
        assert np.array_equal(bits, m.reshape(-1))
        # packed buffer closed form: one run per owned row [rN+1, rN+N-1)
        nr, ne, rs, re, pay = oracle.packed_runs(oracle.pack(bms[g], d2))
        assert nr == b - a and ne == (b - a) * (N - 2)
        assert rs.tolist() == [r * N + 1 for r in range(a, b)]
        assert re.tolist() == [r * N + N - 1 for r in range(a, b)]


def test_sparse_rows_body():
    N = 40
    src = gen.jacobi_field(3, N)
    dst = np.zeros_like(src)
    bms = oracle.sparse_rows(src, dst, 7, P=3, track=True)
    for i in range(N):
        if i % 7 == 0:
            assert np.array_equal(dst[i], src[i] + np.float32(1.0))
        else:
            assert np.all(dst[i] == 0)
    allbits = np.bitwise_or.reduce(bms, axis=0)
    bits = np.unpackbits(allbits.view(np.uint8), bitorder="little")[:N * N].reshape(N, N)
    assert np.array_equal(bits.any(axis=1), np.arange(N) % 7 == 0)


@pytest.mark.parametrize("P", [1, 3])
def test_masked_write_body_brute_force(P):
    n = 1000
    src = gen.u_fill(9, 0, n).astype(np.float32)
    mask = gen.write_mask(10, n, 0.4, 3)
    dst = np.full(n, -5.0, dtype=np.float32)
    bms = oracle.masked_write(src, mask, dst, P=P, track=True)
    bounds = [((g * n) // P, ((g + 1) * n) // P) for g in range(P)]   # L108 chunks, by hand
    for e in range(n):
        exp = float(np.float32(src[e]) + np.float32(1.0)) if mask[e] else -5.0
        assert float(dst[e]) == exp
        for g, (a, b) in enumerate(bounds):
            bit = (int(bms[g][e // 32]) >> (e % 32)) & 1
            assert bit == (1 if (mask[e] and a <= e < b) else 0)


def test_write_mask_recipe():
    m = gen.write_mask(3, 1000, 0.5, 7)
    assert m.size == 1000 and set(np.unique(m)) <= {0, 1}
    assert all(len(set(m[s:s + 7])) == 1 for s in range(0, 1000, 7))   # constant on segments
    assert 0.3 < m.mean() < 0.7
    assert gen.write_mask(3, 100, 1.0).all() and not gen.write_mask(3, 100, 0.0).any()


# ---- GEMM -------------------------------------------------------------------------------------
def _bf16(x):
    return (np.asarray(x, dtype=np.float32).view(np.uint32) >> 16).astype(np.uint16)


def test_gemm_identity():
    A = gen.bf16_matrix(3, 48, 64, gen.BF16_UNIT)
    I = _bf16(np.eye(64))
    assert np.array_equal(oracle.gemm_rows_f64(A, I, np.arange(48)), gen.bf16_to_f32(A).astype(np.float64))
    I2 = _bf16(np.eye(48))
    assert np.array_equal(oracle.gemm_rows_f64(I2, A, np.arange(48)), gen.bf16_to_f32(A).astype(np.float64))


def test_gemm_rank1_and_small_integers():
    rng = np.random.default_rng(0)
    u, v = rng.integers(-3, 4, 20), rng.integers(-3, 4, 33)
    w, z = rng.integers(-3, 4, 33), rng.integers(-3, 4, 17)
    A, B = np.outer(u, v), np.outer(w, z)
    got = oracle.gemm_rows_f64(_bf16(A), _bf16(B), np.arange(20))
    assert np.array_equal(got, (int(v @ w) * np.outer(u, z)).astype(np.float64))
    Ai = gen.bf16_matrix(3, 31, 45, gen.BF16_INTS)
    Bi = gen.bf16_matrix(4, 45, 29, gen.BF16_INTS)
    ia = gen.bf16_to_f32(Ai).astype(np.int64)
    ib = gen.bf16_to_f32(Bi).astype(np.int64)
    rows = np.array([0, 7, 30])
    assert np.array_equal(oracle.gemm_rows_f64(Ai, Bi, rows), (ia @ ib)[rows].astype(np.float64))


def test_gemm_unit_inputs_vs_exact_rationals():
    A = gen.bf16_matrix(3, 4, 40, gen.BF16_UNIT)
    B = gen.bf16_matrix(4, 40, 5, gen.BF16_UNIT)
    fa, fb = gen.bf16_to_f32(A), gen.bf16_to_f32(B)
    got = oracle.gemm_rows_f64(A, B, np.arange(4))
    for i in range(4):
        for j in range(5):
            exact = sum(Fraction(float(fa[i, k])) * Fraction(float(fb[k, j])) for k in range(40))
            assert abs(got[i, j] - float(exact)) <= 40 * 2.0 ** -52 * float(exact)


# ---- k-means (readings in DESIGN.md) ------------------------------------------------------------
def test_kmeans_lattice_closed_form():
    n, d, k = 4096, 16, 32
    x, lab, _ = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
    cen, member = oracle.kmeans_run(x, k, 1)
    assert np.array_equal(member, lab)                  # iteration 1 recovers the true labels
    for c in range(k):                                  # centroids = exact means, fp64 then fp32
        pts = x[lab == c].astype(np.float64)
        for j in range(d):
            exact = sum(Fraction(float(v)) for v in pts[:, j]) / len(pts)
            assert cen[c, j] == np.float32(float(exact))
    cen20, member20 = oracle.kmeans_run(x, k, 20)       # iterations 2..20 are stationary
    assert np.array_equal(cen20, cen) and np.array_equal(member20, lab)


def test_kmeans_assign_integer_brute_force():
    rng = np.random.default_rng(5)
    x = rng.integers(-6, 7, (300, 5)).astype(np.float32)
    cen = rng.integers(-6, 7, (9, 5)).astype(np.float32)
    m = oracle.kmeans_assign(x, cen)
    for p in range(300):
        d2 = [int(((x[p].astype(int) - cen[c].astype(int)) ** 2).sum()) for c in range(9)]
        assert m[p] == d2.index(min(d2))                  # exact distances; ties -> lowest index


def test_kmeans_ties_and_empty_cluster():
    x = np.array([[0, 0], [10, 10], [0, 1], [10, 9]], dtype=np.float32)
    cen = np.array([[0, 0], [0, 0], [10, 10]], dtype=np.float32)     # duplicate centroid 0 == 1
    m = oracle.kmeans_assign(x, cen)
    assert m.tolist() == [0, 2, 0, 2]                    # lowest index wins the tie
    newc = cen.copy()
    s, c = oracle.kmeans_update(x, m, newc)
    assert c.tolist() == [2, 0, 2]
    assert newc[1].tolist() == [0, 0]                    # empty cluster keeps its value
    assert newc[0].tolist() == [0, 0.5] and newc[2].tolist() == [10, 9.5]


def test_kmeans_thread_invariance():
    x = gen.kmeans_points(5, 20000, 16, 64, gen.KM_OVERLAP)
    c1, m1 = oracle.kmeans_run(x, 64, 3, nthreads=1)
    c2, m2 = oracle.kmeans_run(x, 64, 3, nthreads=4)
    assert np.array_equal(c1, c2) and np.array_equal(m1, m2)


def test_dependence_cone_window_reproduces_full_field():
    """Pins the sampled full-size parity method of tests/test_gpu_fullsize.py: after S sweeps a
    point depends only on the initial field within distance S, so sweeping the sub-grid of radius
    S+1 around it (true boundaries kept) reproduces the full-field value bit for bit."""
    from tests.test_gpu_fullsize import _oracle_point_window
    N, S = 200, 7
    A = gen.jacobi_field(2, N)
    B = A.copy()
    oracle.jacobi_run(A, B, S)
    for (i, j) in [(1, 1), (N - 2, N - 2), (50, 100), (1, N - 2), (100, 1), (8, 8)]:
        F, G, i0, j0 = _oracle_point_window(2, N, S, i, j)
        assert A[i, j] == F[i - i0, j - j0] and B[i, j] == G[i - i0, j - j0]


# ---- irregular writes (write misses, L137) ------------------------------------------------------
def test_scatter_pins():
    n = 1000
    src = np.arange(n, dtype=np.float32) * np.float32(0.5)
    ident = np.arange(n, dtype=np.int32)
    dst = np.zeros(n, np.float32)
    miss = oracle.scatter(src, ident, dst, P=4)
    assert np.array_equal(dst, src) and miss.tolist() == [0, 0, 0, 0]   # no write leaves its window
    rev = ident[::-1].copy()
    dst2 = np.zeros(n, np.float32)
    miss2 = oracle.scatter(src, rev, dst2, P=2)
    assert np.array_equal(dst2, src[::-1]) and miss2.tolist() == [500, 500]  # every write crosses
    perm = gen.permutation(9, n)
    assert np.array_equal(np.sort(perm), ident)                           # a permutation
    d3 = np.zeros(n, np.float32)
    oracle.scatter(src, perm, d3)
    inv = np.empty(n, np.int32)
    inv[perm] = ident                                                      # inverse permutation
    back = np.zeros(n, np.float32)
    oracle.scatter(d3, inv, back)
    assert np.array_equal(back, src)
    # brute-force miss counts at P=3
    m3 = oracle.scatter(src, perm, np.zeros(n, np.float32), P=3)
    for g in range(3):
        a, b = oracle.partition(0, n, 3, g)
        assert m3[g] == sum(1 for i in range(a, b) if not (a <= perm[i] < b))


# ---- 3-D 7-point Jacobi (row f2) ------------------------------------------------------------------
def _sweeps3(A, S):
    A = A.copy()
    B = A.copy()
    oracle.jacobi3d_run(A, B, S)
    return A if S % 2 == 0 else B


def test_jacobi3d_fixed_points_and_reflections():
    c = np.full((9, 10, 12), 3.0, np.float32)
    assert np.array_equal(_sweeps3(c, 6), c)                       # constant field
    i, j, k = np.meshgrid(np.arange(9), np.arange(10), np.arange(12), indexing="ij")
    lin = (2 * i - 3 * j + 5 * k + 7).astype(np.float32)           # harmonic, integer sums exact
    assert np.array_equal(_sweeps3(lin, 6), lin)
    rng = np.random.default_rng(1)
    A = rng.random((8, 9, 12), dtype=np.float32)
    out = _sweeps3(A, 5)
    for ax in range(3):                                            # each pair (a+b) is commutative
        assert np.array_equal(_sweeps3(np.ascontiguousarray(np.flip(A, ax)), 5), np.flip(out, ax))


def test_jacobi3d_dyadic_exact_rationals():
    rng = np.random.default_rng(2)
    A = (rng.integers(0, 16, (6, 5, 7)) / 8.0).astype(np.float32)
    F = A.astype(object)
    F = np.vectorize(lambda v: Fraction(float(v)))(A)
    for s in range(3):
        G = F.copy()
        for i in range(1, 5):
            for j in range(1, 4):
                for k in range(1, 6):
                    G[i, j, k] = (F[i - 1, j, k] + F[i + 1, j, k] + F[i, j - 1, k] + F[i, j + 1, k] +
                                  F[i, j, k - 1] + F[i, j, k + 1] + 2 * F[i, j, k]) / 8
        F = G
        assert np.array_equal(_sweeps3(A, s + 1).astype(np.float64), F.astype(np.float64))
