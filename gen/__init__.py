"""Seeded synthetic input generators (recipe in DESIGN.md §Inputs).

Shared by tests/, bench.py and __graft_entry__.smoke(). Holds none of the
method's arithmetic: only the SplitMix64 counter generator and the workload
value recipes. Backed by gen/libaccgen.so (plain C, OpenMP), built by
__graft_entry__.build() / `make gen`.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

_M64 = (1 << 64) - 1


def u_py(seed: int, i: int) -> int:
    """Pure-Python big-int SplitMix64 draw (independent check of the C generator)."""
    x = (seed * 0x9E3779B97F4A7C15 + (i + 1) * 0xD1B54A32D192ED03) & _M64
    x ^= x >> 30
    x = (x * 0xBF58476D1CE4E5B9) & _M64
    x ^= x >> 27
    x = (x * 0x94D049BB133111EB) & _M64
    x ^= x >> 31
    return x


def lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libaccgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build() or `make gen`")
        L = ctypes.CDLL(path)
        i64, u64, i32, vp = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p
        L.accgen_u.restype = u64
        L.accgen_u.argtypes = [u64, u64]
        L.accgen_u_fill.argtypes = [u64, u64, i64, vp]
        L.accgen_jacobi_rows.argtypes = [u64, i64, i64, i64, vp, i32]
        L.accgen_bf16_matrix.argtypes = [u64, i64, i64, i64, i64, i32, vp, i32]
        L.accgen_kmeans_centres.argtypes = [u64, i32, i32, i32, vp]
        L.accgen_kmeans_points.argtypes = [u64, i64, i32, i32, i32, vp, i64, i64, vp, vp, i32]
        L.accgen_permutation.argtypes = [u64, i64, vp]
        L.accgen_field3d.argtypes = [u64, i64, i64, i64, i64, i64, vp, i32]
        _LIB = L
    return _LIB


def _ptr(a) -> int:
    """Address of a numpy array or a CPU torch tensor (pinned buffers are torch tensors)."""
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def u(seed: int, i: int) -> int:
    return int(lib().accgen_u(seed, i))


def u_fill(seed: int, i0: int, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint64)
    lib().accgen_u_fill(seed, i0, n, out.ctypes.data)
    return out


def jacobi_field(seed: int, N: int, r0: int = 0, r1: int | None = None, out=None, nthreads: int = 0):
    """Rows [r0, r1) of the N x N Jacobi field (row 0 = 1, other boundary 0, interior U[0,1))."""
    r1 = N if r1 is None else r1
    if out is None:
        out = np.empty((r1 - r0, N), dtype=np.float32)
    lib().accgen_jacobi_rows(seed, N, r0, r1, _ptr(out), nthreads)
    return out


BF16_INTS, BF16_UNIT, BF16_SIGNED = 0, 1, 2


def bf16_matrix(seed: int, rows: int, cols: int, kind: int, r0: int = 0, r1: int | None = None,
                out=None, nthreads: int = 0):
    """bf16 bit patterns (uint16) of rows [r0, r1) of a rows x cols matrix."""
    r1 = rows if r1 is None else r1
    if out is None:
        out = np.empty((r1 - r0, cols), dtype=np.uint16)
    lib().accgen_bf16_matrix(seed, rows, cols, r0, r1, kind, _ptr(out), nthreads)
    return out


KM_LATTICE, KM_OVERLAP = 0, 1


def kmeans_centres(seed: int, k: int, d: int, mode: int) -> np.ndarray:
    out = np.empty((k, d), dtype=np.float32)
    lib().accgen_kmeans_centres(seed, k, d, mode, out.ctypes.data)
    return out


def kmeans_points(seed: int, n: int, d: int, k: int, mode: int, p0: int = 0, p1: int | None = None,
                  out=None, labels: bool = False, nthreads: int = 0):
    """Points [p0, p1) of the k-means set (and their generating labels if labels=True)."""
    p1 = n if p1 is None else p1
    cen = kmeans_centres(seed, k, d, mode)
    if out is None:
        out = np.empty((p1 - p0, d), dtype=np.float32)
    lab = np.empty(p1 - p0, dtype=np.int32) if labels else None
    lib().accgen_kmeans_points(seed, n, d, k, mode, cen.ctypes.data, p0, p1, _ptr(out),
                               lab.ctypes.data if labels else None, nthreads)
    return (out, lab, cen) if labels else out


def field3d(seed: int, n0: int, n1: int, n2: int, i0: int = 0, i1: int | None = None, out=None,
            nthreads: int = 0):
    """Planes [i0, i1) of the 3-D Jacobi field (plane 0 = 1, other faces 0, interior U[0,1))."""
    i1 = n0 if i1 is None else i1
    if out is None:
        out = np.empty((i1 - i0, n1, n2), dtype=np.float32)
    lib().accgen_field3d(seed, n0, n1, n2, i0, i1, _ptr(out), nthreads)
    return out


def permutation(seed: int, n: int) -> np.ndarray:
    """Seeded random permutation of [0, n) as int32 (index array of the scatter workload)."""
    out = np.empty(n, dtype=np.int32)
    lib().accgen_permutation(seed, n, out.ctypes.data)
    return out


def write_mask(seed: int, n: int, density: float, run: int = 1) -> np.ndarray:
    """uint8 mask of n elements in segments of `run` elements: segment s is set iff
    (u(seed, s) >> 40) < density * 2^24 (so density 1 sets everything, 0 nothing)."""
    nseg = (n + run - 1) // run
    thr = int(density * (1 << 24))
    seg = ((u_fill(seed, 0, nseg) >> np.uint64(40)) < np.uint64(thr)).astype(np.uint8)
    return np.repeat(seg, run)[:n].copy()


def bf16_to_f32(a: np.ndarray) -> np.ndarray:
    """Exact widening of bf16 bit patterns to fp32 (a bit shift, no rounding)."""
    return (a.astype(np.uint32) << 16).view(np.float32)


def kmeans_points_real(seed: int, n: int, d: int, k: int) -> np.ndarray:
    """Real-valued k-means input in the style of the paper's KMEANS data (kddcup feature vectors,
    Table II): arbitrary fp32 values, not on any fixed-point grid. Per dimension a kind is drawn:
    non-negative counts (integers, heavy tailed), rates in [0, 1] (full 24-bit mantissas), or
    signed real values with magnitudes spread over ~40 binades; points scatter multiplicatively
    around k seeded centres; about 10 % of the values are zero. Seeded numpy PCG64."""
    rng = np.random.default_rng(seed)
    kinds = rng.integers(0, 3, d)
    centres = np.empty((k, d))
    for j in range(d):
        if kinds[j] == 0:
            centres[:, j] = np.floor(rng.lognormal(3.0, 2.0, k))
        elif kinds[j] == 1:
            centres[:, j] = rng.random(k)
        else:
            centres[:, j] = rng.choice([-1.0, 1.0], k) * 2.0 ** rng.uniform(-20, 20, k)
    lab = rng.integers(0, k, n)
    x = centres[lab] * (1.0 + 0.05 * rng.standard_normal((n, d)))
    for j in range(d):
        if kinds[j] == 0:
            x[:, j] = np.floor(np.abs(x[:, j]))
        elif kinds[j] == 1:
            x[:, j] = np.clip(x[:, j], 0.0, 1.0)
    x[rng.random((n, d)) < 0.1] = 0.0
    return np.ascontiguousarray(x.astype(np.float32))
