"""One k-means assign loop at 2^24 points (C4 shape) for an ncu capture of the assign kernel."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A
from paper_conf_icpp_komodamnm13_b200 import workloads as WL
n, d, k = 1 << 24, 16, 256
x = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE)
cen = np.ascontiguousarray(x[:k]).copy()
member = np.zeros(n, dtype=np.int32); sums = np.zeros((k, d), dtype=np.int64); cnt = np.zeros(k, dtype=np.int64)
A.accmg_init(num_partitions=1, device=0)
regs = [A.accmg_region_create(a) for a in (x, cen, member, sums, cnt)]
for _ in range(3):
    WL.kmeans_loops(*regs, n, d, k)
A.accmg_barrier()
A.accmg_finalize()
