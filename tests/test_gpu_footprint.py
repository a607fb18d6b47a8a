"""§8 row f4 / Fig. 9 (L249-252): with localaccess declarations each partition allocates only the
sub-array it accesses, so the total User memory of a distributed array does not grow with the
partition count; without declarations every partition holds a full replica."""
import numpy as np
import pytest

import gen
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_user_memory_declared_vs_undeclared(P):
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N = 1024
    arr = N * N * 4
    for declared in (True, False):
        A0 = gen.jacobi_field(2, N)
        A, B = A0.copy(), A0.copy()
        with runtime(num_partitions=P) as acc:
            rA, rB = acc.accmg_region_create(A), acc.accmg_region_create(B)
            for s in range(3):
                WL.jacobi_sweep(rA, rB, s, N, declared)
            st = acc.accmg_get_stats()
        user = st["device_bytes_user"]
        if declared:
            # 2 arrays, each split into P windows + halo rows and one row of allocation padding
            # on each side (ensure_alloc pads new hulls by one declared stride)
            assert user <= 2 * arr + 2 * 4 * P * N * 4
            assert user >= 2 * arr
        else:
            assert user == 2 * arr * P                 # full replicas (L121 replica policy)
            if P > 1:                                  # one partition: nothing to keep coherent
                assert st["device_bytes_system"] >= 2 * P * arr // 32   # L1 dirty bitmaps
