"""GPU parity of the deep-halo Jacobi body (§8 row f2: h > 1 halos, one exchange per h sweeps,
redundant compute of the halo rows) through the C ABI vs the oracle's single sweeps.

Bit-exact: h sweeps per loop perform the same fp32 operations in the same order as h
single-sweep loops (DESIGN.md f2), so the arrays must equal the oracle's after every schedule."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _oracle(A0, loops, h):
    """x_j = J^(h j)(A0); after `loops` loops A holds x_L (L even) or x_(L-1), B the other."""
    xs = [A0.copy()]
    cur = A0.copy()
    tmp = A0.copy()
    for _ in range(loops):
        for _ in range(h):
            oracle.jacobi_sweep(cur, tmp, nthreads=0)
            cur, tmp = tmp, cur
        xs.append(cur.copy())
    last, prev = xs[loops], xs[loops - 1] if loops > 0 else A0
    return (last, prev) if loops % 2 == 0 else (prev, last)


def _gpu(A0, loops, h, P, **kw):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    A, B = A0.copy(), A0.copy()
    with runtime(num_partitions=P, **kw) as acc:
        WL.jacobi_deep_run(A, B, loops * h, h)
        st = acc.accmg_get_stats()
    return A, B, st


@pytest.mark.parametrize("P", [1, 2, 3, 8])
@pytest.mark.parametrize("h", [1, 2, 4, 8])
def test_deep_bitexact(P, h):
    N, loops = 512, 3
    A0 = gen.jacobi_field(11, N)
    oA, oB = _oracle(A0, loops, h)
    A, B, st = _gpu(A0, loops, h, P)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    if P > 1:
        # the loops after the first read h halo rows per side per internal partition boundary
        assert st["bytes_declared"] == (loops - 1) * 2 * (P - 1) * h * N * 4


@pytest.mark.parametrize("N,P,h", [(5, 2, 2), (37, 8, 6), (130, 5, 3), (257, 7, 16), (64, 8, 12)])
def test_deep_ragged_and_halo_wider_than_chunk(N, P, h):
    """Halo deeper than a partition's chunk (windows spanning several owners) and ragged sizes."""
    A0 = gen.jacobi_field(12, N)
    A0[:, 0] = 0.5
    A0[:, -1] = -0.25
    oA, oB = _oracle(A0, 2, h)
    A, B, _ = _gpu(A0, 2, h, P)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)


@pytest.mark.parametrize("N,P,h", [(132, 3, 5), (388, 5, 7), (260, 8, 8), (128, 8, 6), (1000, 2, 2), (644, 1, 3)])
def test_fused_shapes_bitexact(N, P, h):
    """Shapes the fused shared-memory kernel takes (cols % 4 == 0, cols >= 128, h <= 8): ragged
    last row/column tiles, partitions shorter than a 64-row tile, halo columns at the domain edge."""
    A0 = gen.jacobi_field(15, N)
    A0[:, 0] = 0.5
    A0[:, -1] = -0.25
    A0[-1, :] = 2.0
    oA, oB = _oracle(A0, 3, h)
    A, B, st = _gpu(A0, 3, h, P)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    if P == 1:  # fused: one kernel per loop (no scratch sweeps, no frame copies)
        assert st["kernel_launches"] == 3, st["kernel_launches"]


def test_deep_equals_single_sweep_schedule():
    """The deep body and h single-sweep loops give the same bits (redundant compute is exact)."""
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N, h, P = 768, 4, 4
    A0 = gen.jacobi_field(13, N)
    A1, B1 = A0.copy(), A0.copy()
    with runtime(num_partitions=P):
        WL.jacobi_run(A1, B1, 2 * h)
    A, B, _ = _gpu(A0, 2, h, P)
    assert np.array_equal(A, A1)


def test_deep_undeclared_tracked():
    """Without localaccess the dst writes are dirty-tracked (L133) and the src replicated."""
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N, h, P = 256, 3, 3
    A0 = gen.jacobi_field(14, N)
    oA, oB = _oracle(A0, 2, h)
    A, B = A0.copy(), A0.copy()
    with runtime(num_partitions=P):
        WL.jacobi_deep_run(A, B, 2 * h, h, declared=False)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
