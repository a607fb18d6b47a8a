"""Drivers of the paper's workload loops through the C ABI (configs C1-C5 of BASELINE.json).

Each driver issues the same sequence of accmg_* calls an OpenACC program annotated with the
paper's directives would make (L81-93 §III.C): regions = data-region arrays, one
accmg_loop_launch per `parallel loop`, declared windows = `localaccess`, REDUCE_SUM =
`reductiontoarray`. Pure marshalling: all computation happens in libaccmg.so.
"""
from __future__ import annotations

import numpy as np

from . import accmg as A


def jacobi_descs(src, dst, N: int, declared: bool):
    """`localaccess` of the 5-point stencil on row-major N x N: iteration i reads rows i-1..i+1
    (stride N, left = right = N) and writes row i (stride N) — L87 with reading G23."""
    return [A.access(src, A.R, declared, N, N, N), A.access(dst, A.W, declared, N, 0, 0)]


def jacobi_sweep(rA, rB, s: int, N: int, declared: bool) -> None:
    src, dst = (rA, rB) if s % 2 == 0 else (rB, rA)
    A.accmg_loop_launch(A.bounds([1, 1], [N - 1, N - 1]), A.BODY_JACOBI2D_5PT, jacobi_descs(src, dst, N, declared),
                        A.accmg_args_jacobi2d(N, N))


def jacobi_run(Ahost: np.ndarray, Bhost: np.ndarray, sweeps: int, declared: bool = True, per_loop_stats: bool = False):
    """S sweeps A -> B -> A ... on an initialised runtime; host arrays are updated at the end.
    Returns the list of per-loop stats deltas if per_loop_stats."""
    N = Ahost.shape[0]
    rA, rB = A.accmg_region_create(Ahost), A.accmg_region_create(Bhost)
    per = []
    try:
        prev = A.accmg_get_stats() if per_loop_stats else None
        for s in range(sweeps):
            jacobi_sweep(rA, rB, s, N, declared)
            if per_loop_stats:
                cur = A.accmg_get_stats()
                per.append({k: cur[k] - prev[k] for k in cur})
                prev = cur
        A.accmg_sync_to_host(rA)
        A.accmg_sync_to_host(rB)
    finally:
        A.accmg_region_destroy(rA)
        A.accmg_region_destroy(rB)
    return per


def jacobi_deep_descs(src, dst, N: int, h: int, declared: bool = True):
    """Deep halos (§8 f2): h sweeps per loop need rows i-h..i+h (stride N, left = right = h*N)."""
    return [A.access(src, A.R, declared, N, h * N, h * N), A.access(dst, A.W, declared, N, 0, 0)]


def jacobi_deep_loop(rA, rB, s: int, N: int, h: int, declared: bool = True) -> None:
    """Loop s of a deep-halo run: dst = J^h(src), alternating A -> B -> A."""
    src, dst = (rA, rB) if s % 2 == 0 else (rB, rA)
    A.accmg_loop_launch(A.bounds([1, 1], [N - 1, N - 1]), A.BODY_JACOBI2D_DEEP,
                        jacobi_deep_descs(src, dst, N, h, declared), A.accmg_args_jacobi2d_deep(N, N, h))


def jacobi_deep_run(Ahost: np.ndarray, Bhost: np.ndarray, sweeps: int, h: int, declared: bool = True):
    """`sweeps` Jacobi sweeps (a multiple of h) as sweeps/h deep-halo loops; the result lands in
    Ahost when sweeps/h is even, else in Bhost (as jacobi_run with sweeps/h sweeps)."""
    if sweeps % h:
        raise ValueError("sweeps must be a multiple of h")
    N = Ahost.shape[0]
    rA, rB = A.accmg_region_create(Ahost), A.accmg_region_create(Bhost)
    try:
        for s in range(sweeps // h):
            jacobi_deep_loop(rA, rB, s, N, h, declared)
        A.accmg_sync_to_host(rA)
        A.accmg_sync_to_host(rB)
    finally:
        A.accmg_region_destroy(rA)
        A.accmg_region_destroy(rB)


def kmeans_loops(rx, rcen, rmem, rsum, rcnt, n: int, d: int, k: int, shift: int = 8) -> None:
    """One k-means iteration = the paper's 2 parallel loops (Table II: KMEANS has 2 loops)."""
    args = A.accmg_args_kmeans(n, d, k, shift, 0)
    A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_KMEANS_ASSIGN,
                        [A.access(rx, A.R, True, d, 0, 0), A.access(rcen, A.R), A.access(rmem, A.W, True, 1, 0, 0),
                         A.access(rsum, A.REDUCE_SUM), A.access(rcnt, A.REDUCE_SUM)], args)
    A.accmg_loop_launch(A.bounds([0], [k]), A.BODY_KMEANS_UPDATE,
                        [A.access(rsum, A.RW), A.access(rcnt, A.RW), A.access(rcen, A.W)], args)


def kmeans_run(x: np.ndarray, k: int, iters: int, shift: int = 8):
    """Rodinia-style k-means (centroids start at the first k points). Returns (centroids, member).
    shift = KMEANS_EXACT: arbitrary finite points (exact sums, centroid = RN64(sum) / count)."""
    n, d = x.shape
    cen = np.ascontiguousarray(x[:k]).copy()
    member = np.zeros(n, dtype=np.int32)
    # exact mode (shift = KMEANS_EXACT): nine int64 windows per (cluster, dim)
    sums = np.zeros((k, d, A.KMEANS_WINDOWS) if shift == A.KMEANS_EXACT else (k, d), dtype=np.int64)
    cnt = np.zeros(k, dtype=np.int64)
    regs = [A.accmg_region_create(a) for a in (x, cen, member, sums, cnt)]
    try:
        for _ in range(iters):
            kmeans_loops(*regs, n, d, k, shift)
        A.accmg_sync_to_host(regs[1])
        A.accmg_sync_to_host(regs[2])
    finally:
        for r in regs:
            A.accmg_region_destroy(r)
    return cen, member


def gemm_descs(rA, rB, rC, M: int, N: int, K: int):
    """A rows declared (stride K), B replicated (no localaccess), C row-block writes (stride N)."""
    return [A.access(rA, A.R, True, K, 0, 0), A.access(rB, A.R), A.access(rC, A.W, True, N, 0, 0)]


def gemm_loop(rA, rB, rC, M: int, N: int, K: int) -> None:
    A.accmg_loop_launch(A.bounds([0, 0], [M, N]), A.BODY_GEMM_BF16_F32, gemm_descs(rA, rB, rC, M, N, K),
                        A.accmg_args_gemm(M, N, K))


def scatter_loop(rsrc, ridx, rdst, n: int, m: int) -> None:
    """One irregular-write loop dst[idx[i]] = src[i]: src and idx distributed by iteration
    (stride 1), dst distributed by owner window (stride 1); misses go through the system buffers."""
    A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_SCATTER,
                        [A.access(rsrc, A.R, True, 1, 0, 0), A.access(ridx, A.R, True, 1, 0, 0),
                         A.access(rdst, A.W, True, 1, 0, 0)], A.accmg_args_scatter(n, m))


def jacobi3d_sweep(rA, rB, s: int, n0: int, n1: int, n2: int, declared: bool) -> None:
    """One 3-D 7-point sweep; planes are the partitioned outer loop: iteration i reads planes
    i-1..i+1 (stride n1*n2, left = right = n1*n2) and writes plane i (L87 on the flattened array)."""
    src, dst = (rA, rB) if s % 2 == 0 else (rB, rA)
    pl = n1 * n2
    A.accmg_loop_launch(A.bounds([1, 1, 1], [n0 - 1, n1 - 1, n2 - 1]), A.BODY_JACOBI3D_7PT,
                        [A.access(src, A.R, declared, pl, pl, pl), A.access(dst, A.W, declared, pl, 0, 0)],
                        A.accmg_args_jacobi3d(n0, n1, n2))


def jacobi3d_run(Ahost, Bhost, sweeps: int, declared: bool = True):
    n0, n1, n2 = Ahost.shape
    rA, rB = A.accmg_region_create(Ahost), A.accmg_region_create(Bhost)
    try:
        for s in range(sweeps):
            jacobi3d_sweep(rA, rB, s, n0, n1, n2, declared)
        A.accmg_sync_to_host(rA)
        A.accmg_sync_to_host(rB)
    finally:
        A.accmg_region_destroy(rA)
        A.accmg_region_destroy(rB)
