"""GPU parity of irregular writes to a distributed array (§8 row f1; L137, L163): writes outside
the writer's declared window are buffered as (index, value) records and completed in the owner's
replica after the kernel. Bit-exact vs the oracle; miss counts equal the oracle's brute force."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _run(src, idx, P, reps=1):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    n = src.size
    dst = np.zeros(n, np.float32)
    with runtime(num_partitions=P) as acc:
        rs, ri, rd = acc.accmg_region_create(src), acc.accmg_region_create(idx), acc.accmg_region_create(dst)
        for _ in range(reps):
            WL.scatter_loop(rs, ri, rd, n, n)
        acc.accmg_sync_to_host(rd)
        st = acc.accmg_get_stats()
    return dst, st


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_permutation_scatter_bitexact(P):
    n = 100003
    src = gen.jacobi_field(3, 317, 0, 317).reshape(-1)[:n].copy()
    idx = gen.permutation(11, n)
    exp = np.zeros(n, np.float32)
    miss = oracle.scatter(src, idx, exp, P=P)
    got, st = _run(src, idx, P)
    assert np.array_equal(got, exp)
    assert st["write_misses"] == int(miss.sum())
    assert st["bytes_write_miss"] == 12 * int(miss.sum())


def test_identity_has_no_misses_and_repeats():
    n = 65536
    src = np.arange(n, dtype=np.float32)
    idx = np.arange(n, dtype=np.int32)
    got, st = _run(src, idx, 4, reps=3)
    assert np.array_equal(got, src) and st["write_misses"] == 0
