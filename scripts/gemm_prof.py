import sys; sys.path.insert(0, '.')
import numpy as np, gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A, workloads as WL
N = 16384
Ab = gen.bf16_matrix(3, N, N, gen.BF16_INTS); Bb = gen.bf16_matrix(4, N, N, gen.BF16_INTS)
C = np.zeros((N, N), np.float32)
A.accmg_init(num_partitions=1, device=0)
ra, rb, rc = A.accmg_region_create(Ab), A.accmg_region_create(Bb), A.accmg_region_create(C)
for _ in range(2): WL.gemm_loop(ra, rb, rc, N, N, N)
A.accmg_barrier(); A.accmg_finalize()
