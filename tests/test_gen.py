"""Generator vectors (T3) and value recipes. CPU only."""
import numpy as np

import gen

T3 = [0x2D0F28C7E7E786B2, 0x3C5B66874B9E8A84, 0x18330D235A79896C, 0x7DA9B98D1AA4DA69]


def test_t3_vectors_c_and_python():
    assert [gen.u(1, i) for i in range(4)] == T3
    assert [gen.u_py(1, i) for i in range(4)] == T3


def test_fill_matches_pointwise():
    a = gen.u_fill(7, 100, 50)
    assert [int(v) for v in a] == [gen.u_py(7, 100 + i) for i in range(50)]


def test_jacobi_field_recipe():
    N = 37
    f = gen.jacobi_field(3, N)
    assert np.all(f[0] == 1.0) and np.all(f[N - 1] == 0.0)
    assert np.all(f[1:N - 1, 0] == 0.0) and np.all(f[1:N - 1, N - 1] == 0.0)
    for (i, j) in [(1, 1), (5, 17), (N - 2, N - 2)]:
        assert f[i, j] == np.float32((gen.u_py(3, i * N + j) >> 40) / 2.0 ** 24)
    inner = f[1:N - 1, 1:N - 1]
    assert inner.min() >= 0.0 and inner.max() < 1.0
    # any row range is generated independently, with any thread count
    part = gen.jacobi_field(3, N, 10, 20, nthreads=3)
    assert np.array_equal(part, f[10:20])


def test_bf16_recipes():
    ints = gen.bf16_matrix(5, 16, 33, gen.BF16_INTS)
    v = gen.bf16_to_f32(ints)
    assert set(np.unique(v).tolist()) <= {-2.0, -1.0, 0.0, 1.0, 2.0}
    assert v[3, 7] == (gen.u_py(5, 3 * 33 + 7) % 5) - 2
    unit = gen.bf16_to_f32(gen.bf16_matrix(5, 16, 33, gen.BF16_UNIT))
    assert unit.min() > 0.0 and unit.max() <= 1.0
    # round-to-nearest-even to bf16 of ((u>>40)+1)*2^-24, computed with exact Python rationals
    from fractions import Fraction
    x = Fraction((gen.u_py(5, 2 * 33 + 4) >> 40) + 1, 2 ** 24)
    e = x.numerator.bit_length() - x.denominator.bit_length()
    if Fraction(2) ** e > x:
        e -= 1
    ulp = Fraction(2) ** (e - 7)
    q, r = divmod(x, ulp)
    q = int(q) + (1 if (r > ulp / 2 or (r == ulp / 2 and int(q) % 2 == 1)) else 0)
    assert unit[2, 4] == float(q * ulp)


def test_kmeans_recipes():
    n, d, k = 3000, 16, 64
    x, lab, cen = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
    assert np.array_equal(lab[:k], np.arange(k))
    assert np.all((x * 256) == np.round(x * 256)) and np.abs(x).max() < 128
    noise = x - cen[lab]
    assert np.abs(noise).max() <= 0.5
    assert np.all((cen + 64) % 16 == 0) and cen.min() >= -64 and cen.max() < 64
    assert len({tuple(c) for c in cen.tolist()}) == k
    x2, lab2, cen2 = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP, labels=True)
    assert np.abs(x2 - cen2[lab2]).max() <= 2.0 and np.all((x2 * 256) == np.round(x2 * 256))
    part = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP, 100, 200, nthreads=2)
    assert np.array_equal(part, x2[100:200])
