#!/usr/bin/env python3
"""The CPU oracle (oracle/oracle.c, as it stands -- never tuned) timed on this host's cores for each
BASELINE.json config, on bounded samples of the same workloads (SURVEY §8.4 "oracle timing").

It is a reported baseline beside the GPU numbers of bench_configs.py, not a target. Each line:
{"config", "unit", "oracle_rate", "threads", "sample", "extrapolated"}; rates are in the configs'
own units (loop iterations per second: Jacobi point updates, GEMM output elements, k-means point
assignments), so GPU / oracle ratios can be read off directly.

  python scripts/oracle_timing.py [--threads 0] [--budget 10]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402


def timed(fn, budget):
    """Runs fn() until `budget` seconds are spent (at least once); returns (calls, seconds)."""
    n, t0 = 0, time.perf_counter()
    while True:
        fn()
        n += 1
        dt = time.perf_counter() - t0
        if dt >= budget:
            return n, dt


def jacobi(cfg, N, sweeps_note, threads, budget):
    if N <= 4096:  # C1: the whole field
        A0 = gen.jacobi_field(1, N)
        A, B = A0.copy(), A0.copy()
        calls, dt = timed(lambda: oracle.jacobi_sweep_rect(A, B, nthreads=threads), budget)
        return {"config": cfg, "unit": "loop iters/s", "oracle_rate": calls * (N - 2) ** 2 / dt,
                "sample": f"{calls} full sweeps of {N}x{N}", "extrapolated": False}
    rows = 4096  # a full-width band of the 32768^2 field (its own Dirichlet frame)
    band = gen.jacobi_field(2, N, 0, rows + 2)
    out = band.copy()
    calls, dt = timed(lambda: oracle.jacobi_sweep_rect(band, out, nthreads=threads), budget)
    return {"config": cfg, "unit": "loop iters/s", "oracle_rate": calls * rows * (N - 2) / dt,
            "sample": f"{calls} sweeps of a {rows + 2}x{N} band ({sweeps_note})", "extrapolated": False}


def gemm(threads, budget):
    N, nrows = 32768, 16  # fp64 oracle rows of the 32768^3 product
    A = gen.bf16_matrix(3, nrows, N, gen.BF16_UNIT)
    B = gen.bf16_matrix(4, N, N, gen.BF16_UNIT)
    rows = np.arange(nrows)
    calls, dt = timed(lambda: oracle.gemm_rows_f64(A, B, rows, nthreads=threads), budget)
    return {"config": "c3", "unit": "loop iters/s (C elements)", "oracle_rate": calls * nrows * N / dt,
            "sample": f"{calls} x {nrows} fp64 rows of C = A.B at N = {N}", "extrapolated": False}


def kmeans(threads, budget):
    n, d, k = 1 << 22, 16, 256
    x = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE)
    cen = np.ascontiguousarray(x[:k]).copy()
    calls, dt = timed(lambda: oracle.kmeans_assign(x, cen, nthreads=threads), budget)
    return {"config": "c4", "unit": "loop iters/s (point assignments)", "oracle_rate": calls * n / dt,
            "sample": f"{calls} assignment passes over 2^22 of the 2^28 points (k = 256, d = 16)",
            "extrapolated": False}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--threads", type=int, default=0, help="OpenMP threads (0 = all host cores)")
    p.add_argument("--budget", type=float, default=10.0, help="seconds per config")
    a = p.parse_args()
    threads = a.threads or len(os.sched_getaffinity(0))
    info = {"host_cores": len(os.sched_getaffinity(0)), "threads": threads}
    try:
        info["cpu_model"] = next(l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name"))
    except Exception:
        pass
    print(json.dumps(info), flush=True)
    for row in (jacobi("c1", 256, "10 sweeps per loop run", threads, a.budget),
                jacobi("c2", 32768, "C2 field", threads, a.budget),
                jacobi("c5", 32768, "C5: same sweep; the oracle has no coherence step", threads, a.budget),
                gemm(threads, a.budget), kmeans(threads, a.budget)):
        row["threads"] = threads
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
