"""Profiling driver: a few deep-halo loops (h from argv, default 8) on a 32768^2 field, P = 1."""
import sys; sys.path.insert(0, '.')
import gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A, workloads as WL
h = int(sys.argv[1]) if len(sys.argv) > 1 else 8
N = 32768
Ah = gen.jacobi_field(2, N); Bh = Ah.copy()
A.accmg_init(num_partitions=1, device=0)
rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
for s in range(3): WL.jacobi_deep_loop(rA, rB, s, N, h)
A.accmg_barrier(); A.accmg_finalize()
