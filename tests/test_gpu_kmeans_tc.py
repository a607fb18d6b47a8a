"""GPU parity of the tensor-core k-means assignment (kmeans_tc.cu: bf16-split x.c on tcgen05, filter
bound, exact fmaf re-check of the candidates) against the oracle's scalar loop, bit-exact, on inputs
chosen to break a filter whose bound is too tight: exact ties everywhere (small-integer points),
points midway between centroids at large magnitude, a wide dynamic range, and every k edge of the
N tiling (1, 31, 32, 33, 255, 256). The default dispatch takes this path for d = 16, k <= 256."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _run(x, k, iters, P=2, shift=8):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    ocen, omem = oracle.kmeans_run(x, k, iters)
    with runtime(num_partitions=P):
        cen, mem = WL.kmeans_run(x, k, iters, shift=shift)
    assert np.array_equal(mem, omem), f"{int((mem != omem).sum())} assignments differ"
    assert np.array_equal(cen, ocen)


def test_small_integer_points_exact_ties():
    """Points in {-2..2}^16: squared distances are small integers, so most points tie between
    several centroids (and the first 256 points contain duplicates): the lowest index must win."""
    rng = np.random.default_rng(11)
    x = rng.integers(-2, 3, (30011, 16)).astype(np.float32)
    x[7] = x[3]
    x[200] = x[3]
    _run(x, 256, 3, P=3, shift=0)


def test_midpoints_at_large_magnitude():
    """Centroids 1000 + {0, 2} (first dimension) and points at 1001 +- m*2^-8: the two distances
    differ by far less than |x|^2 * 2^-16, so both must be candidates and the fmaf chains decide."""
    rng = np.random.default_rng(12)
    k, n = 64, 20000
    base = (rng.integers(-4, 5, (n, 16)) * 16.0 + 1000.0).astype(np.float32)
    x = base.copy()
    x[:k:2, 0] = 1000.0
    x[1:k:2, 0] = 1002.0
    x[1:k:2, 1:] = x[:k:2, 1:]
    x[k:, 0] = 1001.0 + rng.integers(-3, 4, n - k) * np.float32(2.0 ** -8)
    _run(x, k, 1, P=2, shift=8)


def test_wide_dynamic_range():
    """Integer points from 0 to +-2^20 in the same set (per-point bound L1 * Cinf spans 40 bits)."""
    rng = np.random.default_rng(13)
    n = 25000
    mag = 2.0 ** rng.integers(0, 21, (n, 1))
    x = (np.round(rng.uniform(-1, 1, (n, 16)) * mag)).astype(np.float32)
    _run(x, 100, 3, P=2, shift=0)


@pytest.mark.parametrize("k", [1, 31, 32, 33, 128, 129, 160, 200, 255, 256])
def test_k_edges_ragged_n(k):
    n = 7 * 128 + 77
    x = gen.kmeans_points(7, n, 16, max(k, 2), gen.KM_OVERLAP)
    x[5] = x[2]
    _run(x, k, 2, P=2)


def test_fixed_point_near_2_31():
    """Fixed-point values x * 2^shift up to +-(2^31 - 256): the byte-plane reduction (u8 x u8 -> s32
    on the tensor cores, bias 2^31) must still give exact int64 sums."""
    rng = np.random.default_rng(14)
    n = 9000
    x = (rng.integers(-(2 ** 23) + 1, 2 ** 23, (n, 16)) * 1.0).astype(np.float32)  # * 2^8 < 2^31
    x[:, 3] = np.float32(2 ** 23 - 1)
    x[::2, 5] = np.float32(-(2 ** 23) + 1)
    _run(x, 200, 2, P=2, shift=8)


def test_many_tiles_per_cta_k256():
    """Every CTA runs dozens of 128-point tiles (steady state of the TMEM ring, the one-hot and
    operand stages, and every epilogue set's second and later tiles), k = 256: both halves."""
    x = gen.kmeans_points(21, 148 * 128 * 24 + 5, 16, 256, gen.KM_OVERLAP)
    _run(x, 256, 2, P=1)
