"""GPU parity of k-means exact mode (shift = KMEANS_EXACT; reading KM-X): arbitrary
finite fp32 points, the scalar assignment loop and the exact member sums (nine int64 windows per
(cluster, dim), rounded once to double by the update), bit-exact against oracle.kmeans_run_exact
(math.fsum) at several partition counts. Inputs: kddcup-style real-valued features (PAPER.md
Table II KMEANS, L219-226), the C4 shape, cancellation-heavy clusters, subnormals and values
spread over 260 binades, and grid data (where exact mode must equal the fixed-point mode)."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _run(x, k, iters, P):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    with runtime(num_partitions=P) as A:
        return WL.kmeans_run(x, k, iters, shift=A.KMEANS_EXACT)


@pytest.mark.parametrize("P", [1, 2, 3])
def test_real_valued_kddcup_style(P):
    x = gen.kmeans_points_real(41, 20011, 34, 23)
    ocen, omem = oracle.kmeans_run_exact(x, 23, 4)
    cen, mem = _run(x, 23, 4, P)
    assert np.array_equal(mem, omem), f"{int((mem != omem).sum())} assignments differ"
    assert np.array_equal(cen, ocen)


def test_c4_shape_real_valued_many_blocks():
    """d = 16, k = 256 (the C4 shape; the window accumulators no longer fit shared memory, so the
    blocks add into the partition's partials directly), dozens of blocks per SM."""
    x = gen.kmeans_points_real(42, 148 * 256 * 3 + 17, 16, 256)
    ocen, omem = oracle.kmeans_run_exact(x, 256, 2)
    cen, mem = _run(x, 256, 2, 2)
    assert np.array_equal(mem, omem), f"{int((mem != omem).sum())} assignments differ"
    assert np.array_equal(cen, ocen)


def test_cancellation_and_extreme_magnitudes():
    """Clusters whose members cancel at 2^100 around small values (a sequential fp64 sum loses the
    small ones), subnormals, zeros, and magnitudes from 2^-149 to 2^127."""
    rng = np.random.default_rng(43)
    n, d, k = 9000, 6, 5
    x = (rng.standard_normal((n, d)) * 4.0).astype(np.float32)
    big = np.float32(2.0 ** 100)
    x[10:400:2, 0] = big
    x[11:401:2, 0] = -big
    x[500:900, 1] = np.float32(1.4e-45) * rng.integers(1, 9, 400).astype(np.float32)  # subnormals
    x[1000:1100, 2] = np.float32(3.0e38) * rng.choice([-1, 1], 100).astype(np.float32)
    x[rng.random((n, d)) < 0.1] = 0.0
    ocen, omem = oracle.kmeans_run_exact(x, k, 3)
    for P in (1, 4):
        cen, mem = _run(x, k, 3, P)
        assert np.array_equal(mem, omem), f"P={P}: {int((mem != omem).sum())} assignments differ"
        assert np.array_equal(cen.view(np.uint32), ocen.view(np.uint32)), f"P={P}"


def test_grid_data_exact_mode_equals_fixed_point_mode():
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    x = gen.kmeans_points(44, 30011, 16, 40, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, 40, 3)
    cen, mem = _run(x, 40, 3, 2)
    with runtime(num_partitions=2):
        cen2, mem2 = WL.kmeans_run(x, 40, 3, shift=8)
    for c, m in ((cen, mem), (cen2, mem2)):
        assert np.array_equal(m, omem) and np.array_equal(c, ocen)


def test_non_finite_point_is_reported():
    from paper_conf_icpp_komodamnm13_b200 import accmg as Amod
    x = gen.kmeans_points_real(45, 4000, 8, 6)
    x[1234, 3] = np.inf
    with pytest.raises(Amod.AccmgError) as ei:
        _run(x, 6, 1, 1)
    assert ei.value.code == Amod.EDATA


def test_tensor_core_path_extreme_points():
    """d = 16, k <= 256 takes the tensor-core filter in exact mode too: points beyond 2^60 (whose
    x.c could overflow the fp32 accumulation) re-check every centroid, the rest are filtered;
    subnormals, zeros and cancelling 2^90 values in the sums."""
    rng = np.random.default_rng(47)
    n, d, k = 40000, 16, 96
    x = (rng.standard_normal((n, d)) * 2.0 ** rng.integers(-30, 30, (n, 1))).astype(np.float32)
    x[100:2100:2, 3] = np.float32(2.0 ** 90)
    x[101:2101:2, 3] = np.float32(-(2.0 ** 90))
    x[5000:5100, :] *= np.float32(2.0 ** 70)   # beyond 2^60: unfiltered points
    x[7000:7400, 5] = np.float32(1.4e-45) * rng.integers(1, 5, 400).astype(np.float32)
    x[rng.random((n, d)) < 0.05] = 0.0
    ocen, omem = oracle.kmeans_run_exact(x, k, 3)
    cen, mem = _run(x, k, 3, 2)
    assert np.array_equal(mem, omem), f"{int((mem != omem).sum())} assignments differ"
    assert np.array_equal(cen.view(np.uint32), ocen.view(np.uint32))


def test_tensor_core_path_centroids_beyond_2_60():
    """Every centroid coordinate large (> 2^60 after the first update): no point is filtered."""
    rng = np.random.default_rng(48)
    x = (rng.standard_normal((6000, 16)) * np.float32(2.0 ** 80)).astype(np.float32)
    ocen, omem = oracle.kmeans_run_exact(x, 40, 2)
    cen, mem = _run(x, 40, 2, 1)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)
