"""Debug: C4 lattice k-means at size n, P=1: compare assignments with the generator labels and the
centroids with the exact means after `iters` iterations; print mismatch statistics."""
import os, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen
from paper_conf_icpp_komodamnm13_b200 import accmg as A
from paper_conf_icpp_komodamnm13_b200 import workloads as WL
n = int(sys.argv[1]); iters = int(sys.argv[2]) if len(sys.argv) > 2 else 2
d, k = 16, 256
x, lab, _ = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
A.accmg_init(num_partitions=1, device=0)
cen, mem = WL.kmeans_run(x, k, iters)
A.accmg_finalize()
bad = np.nonzero(mem != lab)[0]
print("n", n, "iters", iters, "label mismatches", bad.size, bad[:10], mem[bad[:10]], lab[bad[:10]])
s = np.zeros((k, d)); c = np.bincount(lab, minlength=k).astype(np.float64)
for j in range(d):
    s[:, j] = np.bincount(lab, weights=x[:, j].astype(np.float64), minlength=k)
exp = (s / c[:, None]).astype(np.float32)
dc = np.nonzero((cen != exp).any(1))[0]
print("centroid mismatches", dc.size, dc[:10])
if dc.size:
    i = dc[0]; print(" c", i, cen[i][:4], exp[i][:4], "count", c[i])
