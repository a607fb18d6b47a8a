"""Phase timing of the tensor-core k-means kernel: needs a build of kmeans_tc.cu with the clock64
instrumentation (km_prof[] counters + accmg_km_prof_read, see profiles/r01/kmeans_tc.log); the
default build does not export accmg_km_prof_read."""
import ctypes, os, sys
sys.path.insert(0, '/root/repo')
import numpy as np
import gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A
from paper_conf_icpp_komodamnm13_b200 import workloads as WL
lib = ctypes.CDLL(os.path.join('/root/repo/paper_conf_icpp_komodamnm13_b200', 'libaccmg.so'))
n, d, k = 1 << 24, 16, 256
x = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE)
cen = np.ascontiguousarray(x[:k]).copy()
member = np.zeros(n, dtype=np.int32); sums = np.zeros((k, d), dtype=np.int64); cnt = np.zeros(k, dtype=np.int64)
A.accmg_init(num_partitions=1, device=0)
regs = [A.accmg_region_create(a) for a in (x, cen, member, sums, cnt)]
WL.kmeans_loops(*regs, n, d, k); A.accmg_barrier()
buf = (ctypes.c_ulonglong * 16)()
lib.accmg_km_prof_read(buf)
for _ in range(3): WL.kmeans_loops(*regs, n, d, k)
A.accmg_barrier()
lib.accmg_km_prof_read(buf)
tiles = 3 * (n // 128)
names = ['cv_wait_x','cv_read_x','cv_wait_a','cv_convert','ep_read_x','ep_misc(pre-wait)','ep_wait_d','ep_pass1','ep_mask_recheck','ep_onehot(+member)','ep_wait_o','mma_wait_afull','mma_wait_dempty']
vals = list(buf)
for i,nm in enumerate(names):
    j = {9:10,10:9}.get(i,i) if False else i
    print(f"{nm:22s} {vals[i]/ (tiles/148) / 4:10.1f} cycles per tile per warp")
