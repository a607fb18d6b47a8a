"""GPU parity of the 3-D 7-point Jacobi body (§8 row f2, TMA-staged tiles) vs the oracle:
bit-exact results for any partition count, declared (plane halos) and undeclared (dirty bits)."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _field(shape, seed):
    return gen.field3d(seed, *shape)


@pytest.mark.parametrize("shape,P,declared", [((20, 33, 36), 1, True), ((20, 33, 36), 3, True),
                                              ((67, 40, 200), 4, True), ((37, 19, 132), 2, False),
                                              ((130, 130, 260), 8, True)])
def test_jacobi3d_bitexact(shape, P, declared):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    S = 5
    A0 = _field(shape, 4)
    oA, oB = A0.copy(), A0.copy()
    oracle.jacobi3d_run(oA, oB, S)
    A, B = A0.copy(), A0.copy()
    with runtime(num_partitions=P, dirty_chunk_bytes=4096) as acc:
        WL.jacobi3d_run(A, B, S, declared=declared)
        st = acc.accmg_get_stats()
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    n0, n1, n2 = shape
    if declared and P > 1:
        assert st["bytes_declared"] == (S - 1) * 2 * (P - 1) * 4 * n1 * n2   # one plane each way
