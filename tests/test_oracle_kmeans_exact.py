"""Pins of the oracle's exact-sum k-means update (reading KM-X; PAPER.md L219-226,
L75-77, L89-91): the centroid is the mean of its members, the exact real sum rounded once to
double, divided in fp64, rounded to fp32. Pinned by an independent exact computation
(fractions.Fraction, whose float() is correctly rounded), a cancellation closed form that a
sequential fp64 sum gets wrong, the empty-cluster rule, and agreement with the sequential-fp64 C
oracle where every fp64 partial sum is exact (the 2^-shift grid of reading W4)."""
from fractions import Fraction

import numpy as np

import gen
import oracle


def _fraction_mean(vals):
    s = sum((Fraction(float(v)) for v in vals), Fraction(0))
    return np.float32(float(s) / float(len(vals)))


def test_exact_update_vs_fractions_wide_magnitudes():
    rng = np.random.default_rng(31)
    n, d, k = 600, 5, 7
    mag = 2.0 ** rng.integers(-140, 120, (n, d))
    x = (rng.uniform(-1, 1, (n, d)) * mag).astype(np.float32)
    x[rng.random((n, d)) < 0.05] = 0.0
    x[::37, 2] = np.float32(1.4e-45)  # subnormals
    member = rng.integers(0, k - 1, n).astype(np.int32)  # cluster k-1 stays empty
    cen = rng.standard_normal((k, d)).astype(np.float32)
    keep = cen[k - 1].copy()
    oracle.kmeans_update_exact(x, member, cen)
    for c in range(k - 1):
        rows = x[member == c]
        for j in range(d):
            assert cen[c, j] == _fraction_mean(rows[:, j]), (c, j)
    assert np.array_equal(cen[k - 1], keep)


def test_cancellation_closed_form():
    """Members {2^100, 1, -2^100}: the mean is exactly 1/3; a left-to-right fp64 sum gives 0."""
    x = np.array([[2.0 ** 100], [1.0], [-(2.0 ** 100)]], np.float32)
    cen = np.zeros((1, 1), np.float32)
    oracle.kmeans_update_exact(x, np.zeros(3, np.int32), cen)
    assert cen[0, 0] == np.float32(1.0 / 3.0)
    assert ((2.0 ** 100 + 1.0) - 2.0 ** 100) / 3.0 == 0.0


def test_exact_run_equals_sequential_fp64_on_the_grid():
    x = gen.kmeans_points(8, 6000, 16, 24, gen.KM_OVERLAP)
    c1, m1 = oracle.kmeans_run(x, 24, 4)
    c2, m2 = oracle.kmeans_run_exact(x, 24, 4)
    assert np.array_equal(m1, m2) and np.array_equal(c1, c2)
