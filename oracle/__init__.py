"""ORACLE — TEST INFRASTRUCTURE ONLY.

Plain, slow CPU implementation of one offloaded parallel loop of Komoda et al. (ICPP'13),
over one host copy of every array (oracle/oracle.c via ctypes), plus a brute-force per-element
coherence model (oracle/model.py). Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` legs may import this package; the product package
(paper_conf_icpp_komodamnm13_b200) never does. It shares no code with the product: it imports
only numpy and gen/ (seeded input generators, which hold none of the method's arithmetic).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build() or `make oracle`")
        L = ctypes.CDLL(path)
        i64, i32, vp = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p
        p64 = ctypes.POINTER(ctypes.c_int64)
        L.orc_partition.argtypes = [i64, i64, i32, i32, p64, p64]
        L.orc_owner.argtypes = [i64, i64, i32, i64]
        L.orc_owner.restype = i32
        L.orc_window_iter.argtypes = [i64, i64, i64, i64, p64, p64]
        L.orc_l2_bits.argtypes = [vp, i64, i64, vp]
        L.orc_pack.argtypes = [vp, i64, vp, i64, vp]
        L.orc_pack.restype = i64
        L.orc_unpack.argtypes = [vp, vp, i64]
        L.orc_jacobi_sweep.argtypes = [vp, vp, i64, i32, vp, i32]
        L.orc_jacobi_run.argtypes = [vp, vp, i64, i32, i32]
        L.orc_jacobi_sweep_rect.argtypes = [vp, vp, i64, i64, i32]
        L.orc_sparse_rows.argtypes = [vp, vp, i64, i64, i32, vp]
        L.orc_masked_write.argtypes = [vp, vp, vp, i64, i32, vp]
        L.orc_gemm_rows_f64.argtypes = [vp, vp, i64, i64, i64, vp, i64, vp, i32]
        L.orc_kmeans_assign.argtypes = [vp, i64, i32, i32, vp, vp, i32]
        L.orc_kmeans_update.argtypes = [vp, i64, i32, i32, vp, vp, vp, vp]
        L.orc_kmeans_run.argtypes = [vp, i64, i32, i32, i32, vp, vp, i32]
        L.orc_scatter.argtypes = [vp, vp, vp, i64, i64, i32, vp]
        L.orc_jacobi3d_sweep.argtypes = [vp, vp, i64, i64, i64, i32, vp, i32]
        L.orc_jacobi3d_run.argtypes = [vp, vp, i64, i64, i64, i32, i32]
        _LIB = L
    return _LIB


def _p(a):
    return None if a is None else a.ctypes.data


# ---- task mapping / windows (L108, L87) ----------------------------------------------------
def partition(lo: int, hi: int, P: int, g: int) -> tuple[int, int]:
    a, b = ctypes.c_int64(), ctypes.c_int64()
    lib().orc_partition(lo, hi, P, g, ctypes.byref(a), ctypes.byref(b))
    return a.value, b.value


def owner(lo: int, hi: int, P: int, i: int) -> int:
    return int(lib().orc_owner(lo, hi, P, i))


def window_iter(stride: int, left: int, right: int, i: int) -> tuple[int, int]:
    a, b = ctypes.c_int64(), ctypes.c_int64()
    lib().orc_window_iter(stride, left, right, i, ctypes.byref(a), ctypes.byref(b))
    return a.value, b.value


# ---- dirty bits / packed buffers (L133-135) -------------------------------------------------
def nwords(extent: int) -> int:
    return (extent + 31) // 32


def l2_bits(l1: np.ndarray, extent: int, chunk_elems: int) -> np.ndarray:
    nch = (extent + chunk_elems - 1) // chunk_elems
    out = np.zeros((nch + 31) // 32, dtype=np.uint32)
    lib().orc_l2_bits(l1.ctypes.data, extent, chunk_elems, out.ctypes.data)
    return out


def pack(l1: np.ndarray, values: np.ndarray) -> np.ndarray:
    """Canonical packed buffer of the dirty elements of `values` (flat), as uint8."""
    v = np.ascontiguousarray(values).reshape(-1)
    l1 = np.ascontiguousarray(l1, dtype=np.uint32)
    n = lib().orc_pack(l1.ctypes.data, v.size, v.ctypes.data, v.itemsize, None)
    out = np.empty(n, dtype=np.uint8)
    lib().orc_pack(l1.ctypes.data, v.size, v.ctypes.data, v.itemsize, out.ctypes.data)
    return out


def unpack(packed: np.ndarray, values: np.ndarray) -> None:
    assert values.flags.c_contiguous
    lib().orc_unpack(packed.ctypes.data, values.ctypes.data, values.itemsize)


def packed_runs(packed: np.ndarray):
    hdr = packed[:16].view(np.uint64)
    nr, ne = int(hdr[0]), int(hdr[1])
    rs = packed[16:16 + 8 * nr].view(np.int64)
    re = packed[16 + 8 * nr:16 + 16 * nr].view(np.int64)
    return nr, ne, rs, re, packed[16 + 16 * nr:]


# ---- loop bodies -----------------------------------------------------------------------------
def jacobi_sweep(src: np.ndarray, dst: np.ndarray, P: int = 1, track: bool = False, nthreads: int = 1):
    """One sweep src -> dst in place on dst; returns P dirty bitmaps if track."""
    N = src.shape[0]
    assert src.dtype == np.float32 and dst.dtype == np.float32 and src.flags.c_contiguous
    bms = np.zeros((P, nwords(N * N)), dtype=np.uint32) if track else None
    lib().orc_jacobi_sweep(src.ctypes.data, dst.ctypes.data, N, P, _p(bms), nthreads)
    return bms


def jacobi_sweep_rect(src: np.ndarray, dst: np.ndarray, nthreads: int = 0) -> None:
    rows, cols = src.shape
    lib().orc_jacobi_sweep_rect(src.ctypes.data, dst.ctypes.data, rows, cols, nthreads)


def jacobi_run(A: np.ndarray, B: np.ndarray, S: int, nthreads: int = 1) -> None:
    lib().orc_jacobi_run(A.ctypes.data, B.ctypes.data, A.shape[0], S, nthreads)


def sparse_rows(inp: np.ndarray, out: np.ndarray, period: int, P: int = 1, track: bool = False):
    N = inp.shape[0]
    bms = np.zeros((P, nwords(N * N)), dtype=np.uint32) if track else None
    lib().orc_sparse_rows(inp.ctypes.data, out.ctypes.data, N, period, P, _p(bms))
    return bms


def masked_write(inp: np.ndarray, mask: np.ndarray, out: np.ndarray, P: int = 1, track: bool = False):
    """out[e] = inp[e] + 1 where mask[e] (flat arrays, in place on out); P bitmaps if track."""
    n = inp.size
    assert inp.dtype == np.float32 and out.dtype == np.float32 and mask.dtype == np.uint8
    bms = np.zeros((P, nwords(n)), dtype=np.uint32) if track else None
    lib().orc_masked_write(inp.ctypes.data, mask.ctypes.data, out.ctypes.data, n, P, _p(bms))
    return bms


def gemm_rows_f64(A: np.ndarray, B: np.ndarray, rows, nthreads: int = 0) -> np.ndarray:
    """fp64 rows of A.B for bf16 bit-pattern inputs A [M][K], B [K][N] (uint16)."""
    M, K = A.shape
    K2, N = B.shape
    assert K == K2 and A.dtype == np.uint16 and B.dtype == np.uint16
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.empty((rows.size, N), dtype=np.float64)
    lib().orc_gemm_rows_f64(A.ctypes.data, B.ctypes.data, M, N, K, rows.ctypes.data, rows.size,
                            out.ctypes.data, nthreads)
    return out


def kmeans_assign(x: np.ndarray, cen: np.ndarray, nthreads: int = 0) -> np.ndarray:
    n, d = x.shape
    k = cen.shape[0]
    m = np.empty(n, dtype=np.int32)
    lib().orc_kmeans_assign(x.ctypes.data, n, d, k, np.ascontiguousarray(cen).ctypes.data,
                            m.ctypes.data, nthreads)
    return m


def kmeans_update(x: np.ndarray, member: np.ndarray, cen: np.ndarray):
    """Updates cen in place; returns (sum fp64 [k][d], cnt int64 [k])."""
    n, d = x.shape
    k = cen.shape[0]
    s = np.empty((k, d), dtype=np.float64)
    c = np.empty(k, dtype=np.int64)
    lib().orc_kmeans_update(x.ctypes.data, n, d, k, member.ctypes.data, cen.ctypes.data,
                            s.ctypes.data, c.ctypes.data)
    return s, c


def kmeans_run(x: np.ndarray, k: int, iters: int, nthreads: int = 0):
    n, d = x.shape
    cen = np.empty((k, d), dtype=np.float32)
    m = np.empty(n, dtype=np.int32)
    lib().orc_kmeans_run(x.ctypes.data, n, d, k, iters, cen.ctypes.data, m.ctypes.data, nthreads)
    return cen, m


def kmeans_update_exact(x: np.ndarray, member: np.ndarray, cen: np.ndarray) -> np.ndarray:
    """KMEANS update loop for arbitrary finite fp32 points (Table II; reductiontoarray
    L75-77, L89-91; reading KM-X in DESIGN.md §2): the new centroid is the mean of its members,

        cen[c][j] = (float)( RN64(sum over p in c of x[p][j]) / (double)cnt[c] )   if cnt[c] > 0,

    the exact real sum rounded once to double (math.fsum is correctly rounded), then the fp64
    division and the rounding to fp32; empty clusters keep their centroid. On points for which
    every fp64 partial sum is exact (the 2^-shift grid of reading W4) this is the sequential-fp64
    update of orc_kmeans_update. Updates cen in place; returns the counts."""
    import math
    k, d = cen.shape
    assert np.all(np.isfinite(x)), "exact mode takes finite points"
    cnt = np.bincount(member, minlength=k).astype(np.int64)
    order = np.argsort(member, kind="stable")
    bounds = np.concatenate(([0], np.cumsum(cnt)))
    xs = x[order].astype(np.float64)  # fp32 -> fp64 is exact
    for c in range(k):
        if cnt[c] == 0:
            continue
        rows = xs[bounds[c]:bounds[c + 1]]
        for j in range(d):
            cen[c, j] = np.float32(math.fsum(rows[:, j].tolist()) / float(cnt[c]))
    return cnt


def kmeans_run_exact(x: np.ndarray, k: int, iters: int, nthreads: int = 0):
    """cen[c] = x[c] for c < k, then `iters` x (assignment: orc_kmeans_assign, the scalar fmaf loop;
    update: kmeans_update_exact). Returns (centroids after the last update, member of the last
    assignment)."""
    cen = np.ascontiguousarray(x[:k]).astype(np.float32).copy()
    m = np.zeros(x.shape[0], dtype=np.int32)
    for _ in range(iters):
        m = kmeans_assign(x, cen, nthreads)
        kmeans_update_exact(x, m, cen)
    return cen, m


def scatter(src: np.ndarray, idx: np.ndarray, dst: np.ndarray, P: int = 0):
    """dst[idx[i]] = src[i] in place; returns per-partition write-miss counts if P > 0."""
    miss = np.zeros(max(P, 1), dtype=np.int64)
    lib().orc_scatter(src.ctypes.data, idx.ctypes.data, dst.ctypes.data, 0, src.size, P, miss.ctypes.data)
    return miss[:P] if P > 0 else None


def jacobi3d_sweep(src: np.ndarray, dst: np.ndarray, P: int = 1, track: bool = False, nthreads: int = 0):
    n0, n1, n2 = src.shape
    bms = np.zeros((P, nwords(src.size)), dtype=np.uint32) if track else None
    lib().orc_jacobi3d_sweep(src.ctypes.data, dst.ctypes.data, n0, n1, n2, P, _p(bms), nthreads)
    return bms


def jacobi3d_run(A: np.ndarray, B: np.ndarray, S: int, nthreads: int = 0) -> None:
    n0, n1, n2 = A.shape
    lib().orc_jacobi3d_run(A.ctypes.data, B.ctypes.data, n0, n1, n2, S, nthreads)
