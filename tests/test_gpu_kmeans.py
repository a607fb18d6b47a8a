"""GPU parity of the k-means loops (config C4 shape): assignment + reductiontoarray + update
through the C ABI vs the oracle, bit-exact (assignments and centroids), at several partition
counts and through the NCCL path."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


@pytest.mark.parametrize("P", [1, 3, 8])
def test_overlapping_set_bitexact(P):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n, d, k, iters = 1 << 15, 16, 64, 20
    x = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, k, iters)
    with runtime(num_partitions=P) as acc:
        cen, mem = WL.kmeans_run(x, k, iters)
        st = acc.accmg_get_stats()
    assert np.array_equal(mem, omem)
    assert np.array_equal(cen, ocen)
    assert st["bytes_reduce"] == iters * 2 * (P - 1) * (k * d + k) * 8
    # link bytes per iteration: the merge reads the P-1 other partials (the ring figure above is
    # the algorithmic volume), and the update loop's writes to the replicated centroids (fp32) and
    # sums / counts (int64, reset) are pushed to the P-1 other replicas, payload only
    assert st["bytes_link"] == iters * (P - 1) * ((k * d + k) * 8 + k * d * 4 + (k * d + k) * 8)


def test_lattice_closed_form_and_ragged_n():
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n, d, k = 100003, 16, 256
    x, lab, _ = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
    with runtime(num_partitions=5):
        cen, mem = WL.kmeans_run(x, k, 3)
    assert np.array_equal(mem, lab)
    ocen, _ = oracle.kmeans_run(x, k, 3)
    assert np.array_equal(cen, ocen)


def test_nccl_allreduce_path():
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n, d, k = 20000, 16, 32
    x = gen.kmeans_points(5, n, d, k, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, k, 5)
    with runtime(num_partitions=2, exchange_mode=A.XCHG_NCCL_ALL):
        cen, mem = WL.kmeans_run(x, k, 5)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)


def test_generic_dimension_and_ties():
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    rng = np.random.default_rng(3)
    n, d, k = 5000, 5, 7
    x = (rng.integers(-512, 512, (n, d)) / 64.0).astype(np.float32)
    x[1] = x[0]                                   # duplicate initial centroid -> ties, empty cluster
    ocen, omem = oracle.kmeans_run(x, k, 4)
    with runtime(num_partitions=3):
        cen, mem = WL.kmeans_run(x, k, 4, shift=6)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)


def test_off_grid_input_is_reported():
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    x = gen.kmeans_points(5, 4096, 16, 8, gen.KM_OVERLAP)
    x[100, 3] += np.float32(1e-3)                 # not on the 2^-8 grid
    with runtime(num_partitions=1):
        with pytest.raises(A.AccmgError) as e:
            WL.kmeans_run(x, 8, 1)
        assert e.value.code == A.EDATA


@pytest.mark.parametrize("k", [37, 258, 301, 600])
def test_d16_odd_k_and_k_beyond_constant_memory(k):
    """d = 16: k <= 256 on the tensor cores (odd k), 256 < k <= 512 on the FP32-pipe constant-memory
    kernel (odd and even k), k > 512 on the shared-memory kernel, with duplicated points (ties)."""
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n = 40000
    x = gen.kmeans_points(6, n, 16, k, gen.KM_OVERLAP)
    x[1] = x[0]                                   # duplicate initial centroid -> ties, an empty cluster
    ocen, omem = oracle.kmeans_run(x, k, 3)
    with runtime(num_partitions=2):
        cen, mem = WL.kmeans_run(x, k, 3)
    assert np.array_equal(mem, omem) and np.array_equal(cen, ocen)
