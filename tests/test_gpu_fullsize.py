"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py / bench_configs.py
time, on outputs the oracle can compute one by one.

* C2/C5 (32768^2, 100 sweeps): the value of point (i, j) after S sweeps depends only on the
  initial field within |di| + |dj| <= S, so the oracle sweeping the (2S+3)^2 sub-grid around a
  sample point (as its own field) reproduces that point exactly — bit-exact sampled parity.
* C3 (32768^3 GEMM): sampled rows, incl. the first/last row of every partition, vs the fp64 oracle
  (integer inputs: bit-exact).
* C4 (2^28 x 16, k = 256): closed form (labels recovered, centroids = exact cluster means).
"""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _oracle_point_window(field_seed, N, S, i, j):
    """Oracle sweeps of the sub-grid within distance S+1 of (i, j) (a rectangle, so true boundary
    rows/columns stay fixed exactly as in the full field). Returns (A, B, i0, j0)."""
    r = S + 1
    i0, i1 = max(0, i - r), min(N, i + r + 1)
    j0, j1 = max(0, j - r), min(N, j + r + 1)
    F = np.ascontiguousarray(gen.jacobi_field(field_seed, N, i0, i1)[:, j0:j1])
    G = F.copy()
    for s in range(S):
        if s % 2 == 0:
            oracle.jacobi_sweep_rect(F, G)
        else:
            oracle.jacobi_sweep_rect(G, F)
    return F, G, i0, j0


@pytest.mark.parametrize("P,declared", [(1, True), (2, True), (8, True), (2, False)])
def test_c2_c5_full_size_sampled(P, declared):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N, S = 32768, 100
    Ah = gen.jacobi_field(2, N)
    Bh = Ah.copy()
    with runtime(num_partitions=P):
        WL.jacobi_run(Ah, Bh, S if declared else 10, declared=declared)
    S = S if declared else 10
    half = 1 + (N - 2) // 2
    pts = [(1, 1), (1, N // 3), (half - 1, 5000), (half, 5000), (half + 1, N - 2), (N - 2, N - 2),
           (12345, 23456), (N // 2 + 7, 2)]
    for (i, j) in pts:
        F, G, i0, j0 = _oracle_point_window(2, N, S, i, j)
        assert Ah[i, j] == F[i - i0, j - j0], (P, declared, i, j)
        assert Bh[i, j] == G[i - i0, j - j0], (P, declared, i, j)


def test_c3_full_size_sampled_rows():
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N, P = 32768, 2
    Ab = gen.bf16_matrix(3, N, N, gen.BF16_INTS)
    Bb = gen.bf16_matrix(4, N, N, gen.BF16_INTS)
    C = np.zeros((N, N), dtype=np.float32)
    with runtime(num_partitions=P) as acc:
        ra, rb, rc = acc.accmg_region_create(Ab), acc.accmg_region_create(Bb), acc.accmg_region_create(C)
        WL.gemm_loop(ra, rb, rc, N, N, N)
        acc.accmg_sync_to_host(rc)
    rows = np.array([0, N // 2 - 1, N // 2, N - 1, 127, 128, 20000])
    R = oracle.gemm_rows_f64(Ab, Bb, rows)
    assert np.array_equal(C[rows], R.astype(np.float32))


def test_c4_full_size_closed_form():
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n, d, k = 1 << 28, 16, 256
    x, lab, _ = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
    with runtime(num_partitions=2):
        cen, mem = WL.kmeans_run(x, k, 20)
    assert np.array_equal(mem, lab)
    s = np.zeros((k, d), dtype=np.float64)
    for c0 in range(0, n, 1 << 24):
        c1 = min(n, c0 + (1 << 24))
        for j in range(d):
            s[:, j] += np.bincount(lab[c0:c1], weights=x[c0:c1, j].astype(np.float64), minlength=k)
    cnt = np.bincount(lab, minlength=k).astype(np.float64)
    assert np.array_equal(cen, (s / cnt[:, None]).astype(np.float32))


@pytest.fixture(scope="module")
def t14_oracle():
    """T14's reference: 2^22 overlapping points, k = 256, 20 iterations, run once by the oracle."""
    n, d, k, iters = 1 << 22, 16, 256, 20
    x = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, k, iters)
    return x, ocen, omem


@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_t14_overlapping_2_22_twenty_iterations(t14_oracle, P):
    """T14: 2^22 overlapping points (near-ties occur), k = 256, 20 iterations,
    bit-exact assignments and centroids against the oracle at P = 1, 2, 4, 8."""
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    x, ocen, omem = t14_oracle
    with runtime(num_partitions=P):
        cen, mem = WL.kmeans_run(x, 256, 20)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)


def test_c4_overlapping_parity_2_20():
    """Overlapping clusters, P = 3 (a partition count that does not divide n) — bit-exact."""
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n, d, k, iters = 1 << 20, 16, 256, 4
    x = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, k, iters)
    with runtime(num_partitions=3):
        cen, mem = WL.kmeans_run(x, k, iters)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)
