import sys; sys.path.insert(0, '.')
import numpy as np, gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A, workloads as WL
n = 1024
Ah = gen.field3d(6, n, n, n); Bh = Ah.copy()
A.accmg_init(num_partitions=1, device=0)
rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
for s in range(3): WL.jacobi3d_sweep(rA, rB, s, n, n, n, True)
A.accmg_barrier(); A.accmg_finalize()
