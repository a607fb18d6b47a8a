import sys; sys.path.insert(0, '.')
import numpy as np, gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A, workloads as WL
n = 1 << 24
x = gen.kmeans_points(4, n, 16, 256, gen.KM_LATTICE)
A.accmg_init(num_partitions=1, device=0)
WL.kmeans_run(x, 256, 3)
A.accmg_finalize()
