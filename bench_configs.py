#!/usr/bin/env python3
"""All five BASELINE.json configs on ONE B200 (bench.py is the driver's single-line C2 bench).

Partitions P > 1 are virtual partitions on the one GPU (separate full-extent replicas, exchanges as
device copies / scatter kernels), which exercises and times every coherence step of the multi-GPU
path except the NVLink transfer itself. One JSON line per (config, P) on stdout:

  python bench_configs.py --configs c1,c2,c3,c4,c5 --partitions 1,2,4,8

Each line: loop iterations/s, ms per loop, per-phase CUDA-event times (body / compaction /
exchange), inter-partition bytes per loop and the dominant kernel's roofline fraction; --check
adds the k-means closed-form check (labels and exact means of the generated clusters). Oracle
parity at these sizes lives in tests/test_gpu_fullsize.py (this script never loads the oracle).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import accmg as A  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import workloads as WL  # noqa: E402


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}


def emit(d):
    print(json.dumps(d), flush=True)


def per_loop(st, loops):
    return {"ms_body": st["ms_body"] / loops, "ms_compact": st["ms_compact"] / loops,
            "ms_exchange": st["ms_exchange"] / loops,
            "bytes_interpartition": st["bytes_interpartition"] / loops,
            "bytes_declared": st["bytes_declared"] / loops,
            "bytes_undeclared_payload": st["bytes_undeclared_payload"] / loops,
            "bytes_undeclared_headers": st["bytes_undeclared_headers"] / loops,
            "bytes_paper_protocol": st["bytes_paper_protocol"] / loops,
            "kernel_launches": st["kernel_launches"] / loops}


def wall(fn):
    A.accmg_barrier()
    t0 = time.perf_counter()
    fn()
    A.accmg_barrier()
    return time.perf_counter() - t0


def device_ms(fn):
    """CUDA-event time of fn's launches on the library stream (ms), synchronised on both sides."""
    import torch
    A.accmg_barrier()
    st = torch.cuda.ExternalStream(A.accmg_stream(), device=0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    fn()
    e1.record(st)
    A.accmg_barrier()
    e1.synchronize()
    return e0.elapsed_time(e1)


def jacobi_cfg(name, N, sweeps, P, declared, check, rounds=5):
    """Alternating passes over the same loops, `rounds` times: unprofiled (no events between the
    launches: the loop time on the device) and profiled (the library's per-phase events: body,
    compaction, exchange time per loop). gap_us = the median over rounds of (unprofiled loop time -
    profiled body time) of adjacent passes, so clock drift between passes cancels."""
    Ah = gen.jacobi_field(2 if N > 256 else 1, N)
    Bh = Ah.copy()
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
        s0 = [0]

        def run():
            for _ in range(sweeps):
                WL.jacobi_sweep(rA, rB, s0[0], N, declared)
                s0[0] += 1

        for _ in range(2):
            WL.jacobi_sweep(rA, rB, s0[0], N, declared)
            s0[0] += 1
        A.accmg_set_profile(False)
        t = wall(run)
        loops, bodies, profs, st = [], [], [], None
        for _ in range(rounds):
            A.accmg_set_profile(False)
            loops.append(device_ms(run) / sweeps)
            A.accmg_set_profile(True)
            A.accmg_barrier()
            A.accmg_reset_stats()
            profs.append(device_ms(run) / sweeps)
            st = A.accmg_get_stats()
            bodies.append(st["ms_body"] / sweeps)
        A.accmg_sync_to_host(rA)
        A.accmg_sync_to_host(rB)
    finally:
        A.accmg_finalize()
    pl = per_loop(st, sweeps)
    body_bytes = 8 * (N - 2) * (N - 2) / P  # per partition launch
    body_ms_launch = st["ms_body"] / max(st["body_launches"], 1)
    gaps = sorted((l - b) * 1e3 for l, b in zip(loops, bodies))
    ms_loop = float(np.median(loops))
    out = {"config": name, "P": P, "N": N, "sweeps": sweeps, "rounds": rounds, "declared": declared,
           "iters_per_s": (N - 2) ** 2 / (ms_loop / 1e3), "ms_per_loop": ms_loop,
           "ms_per_loop_wall": t / sweeps * 1e3, "ms_per_loop_profiled": float(np.median(profs)), **pl,
           "gap_us": float(np.median(gaps)), "gap_us_range": [gaps[0], gaps[-1]],
           "body_GBs": body_bytes / (body_ms_launch / 1e3) / 1e9}
    out["body_frac_of_measured_hbm"] = out["body_GBs"] / peaks()["hbm_gbs"]
    return out


def gemm_cfg(N, P, reps, check):
    pk = peaks()
    Ab = gen.bf16_matrix(3, N, N, gen.BF16_INTS)
    Bb = gen.bf16_matrix(4, N, N, gen.BF16_INTS)
    C = np.zeros((N, N), dtype=np.float32)
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        ra, rb, rc = A.accmg_region_create(Ab), A.accmg_region_create(Bb), A.accmg_region_create(C)
        WL.gemm_loop(ra, rb, rc, N, N, N)  # warm-up (and copy-in)
        A.accmg_barrier()
        A.accmg_reset_stats()
        t = wall(lambda: [WL.gemm_loop(ra, rb, rc, N, N, N) for _ in range(reps)])
        st = A.accmg_get_stats()
        A.accmg_sync_to_host(rc)
    finally:
        A.accmg_finalize()
    flop = 2.0 * N ** 3
    ms_launch = st["ms_body"] / max(st["body_launches"], 1)
    out = {"config": "c3", "P": P, "N": N, "reps": reps, "iters_per_s": N * N * reps / t,
           "ms_per_loop": t / reps * 1e3, **per_loop(st, reps),
           "tflops": flop * reps / t / 1e12, "body_tflops_per_launch": flop / P / (ms_launch / 1e3) / 1e12}
    out["frac_of_measured_bf16_burst"] = out["tflops"] / pk["bf16_tflops"]
    out["frac_of_measured_bf16_sustained"] = out["tflops"] / pk.get("bf16_tflops_sustained", pk["bf16_tflops"])
    return out


def kmeans_cfg(n, iters, P, check, exact=False):
    d, k = 16, 256
    pk = peaks()
    t0 = time.perf_counter()
    x, lab, _ = gen.kmeans_points(4, n, d, k, gen.KM_LATTICE, labels=True)
    tgen = time.perf_counter() - t0
    cen = np.ascontiguousarray(x[:k]).copy()
    member = np.zeros(n, dtype=np.int32)
    shift = A.KMEANS_EXACT if exact else 8  # exact mode: the general-data path (nine windows per sum)
    sums = np.zeros((k, d, A.KMEANS_WINDOWS) if exact else (k, d), dtype=np.int64)
    cnt = np.zeros(k, dtype=np.int64)
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        regs = [A.accmg_region_create(a) for a in (x, cen, member, sums, cnt)]
        WL.kmeans_loops(*regs, n, d, k, shift)  # iteration 1 (copy-in) untimed
        A.accmg_barrier()
        A.accmg_reset_stats()
        t = wall(lambda: [WL.kmeans_loops(*regs, n, d, k, shift) for _ in range(iters - 1)])
        st = A.accmg_get_stats()
        A.accmg_sync_to_host(regs[1])
        A.accmg_sync_to_host(regs[2])
    finally:
        A.accmg_finalize()
    its = iters - 1
    ms_assign = st["ms_body"] / its  # body time includes the (tiny) update loop
    out = {"config": "c4x" if exact else "c4", "P": P, "n": n, "iters_timed": its, "iters_per_s": n * its / t,
           "ms_per_iteration": t / its * 1e3, **per_loop(st, 2 * its), "gen_s": tgen}
    impl = "exact" if exact else ("tc" if k <= 256 else "fp32")
    # HBM view: 64 B of point coordinates read + 4 B of assignment written per point
    out["assign_hbm_gbs"] = n * (d * 4 + 4) / (ms_assign / 1e3) / 1e9
    out["assign_frac_of_measured_hbm"] = out["assign_hbm_gbs"] / pk["hbm_gbs"]
    if impl == "tc":
        # tensor-pipe view of the tcgen05 formulation (kmeans_tc.cu): per 128-point tile 8 distance
        # MMAs (M=128, N=128, K=16 bf16: 64 cycles each) + 8 reductiontoarray MMAs (M=128, N=32,
        # K=32 u8 at twice the bf16 rate: 16 cycles each) = 640 tensor cycles per tile per SM at
        # 1.965 GHz (round 1's formulation, with 32-bit reduction words, was 768)
        tiles = -(-n // 128)
        t_tensor = tiles / 148 * 640 / 1.965e9
        out["assign_tensor_bound_ms"] = t_tensor * 1e3
        out["assign_frac_of_tensor_bound"] = t_tensor / (ms_assign / 1e3)
    else:
        # FP32-pipe kernels: 2 k d lane-ops per point (1 sub + 1 fma) against 148 SMs x 128 lanes
        out["fp32_lane_ops_per_s"] = 2.0 * n * k * d / (ms_assign / 1e3)
        out["frac_of_fp32_lane_peak_1965MHz"] = out["fp32_lane_ops_per_s"] / (148 * 128 * 1.965e9)
    out["kmeans_impl"] = impl
    if check:
        ok = np.array_equal(member, lab)
        # closed form: centroids are the exact means of the generated clusters
        s = np.zeros((k, d), dtype=np.float64)
        for c0 in range(0, n, 1 << 24):
            c1 = min(n, c0 + (1 << 24))
            for j in range(d):
                s[:, j] += np.bincount(lab[c0:c1], weights=x[c0:c1, j].astype(np.float64), minlength=k)
        c = np.bincount(lab, minlength=k).astype(np.float64)
        ok = ok and np.array_equal(cen, (s / c[:, None]).astype(np.float32))
        out["parity"] = "closed-form labels+means" if ok else "MISMATCH"
    return out


def jacobi3d_cfg(n, sweeps, P, declared=True):
    """§8 row f2: 3-D 7-point Jacobi on n^3 fp32, plane-block partition, TMA-staged tiles."""
    Ah = gen.field3d(6, n, n, n)
    Bh = Ah.copy()
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
        for s in range(2):
            WL.jacobi3d_sweep(rA, rB, s, n, n, n, declared)
        A.accmg_barrier()
        A.accmg_reset_stats()
        t = wall(lambda: [WL.jacobi3d_sweep(rA, rB, s, n, n, n, declared) for s in range(2, 2 + sweeps)])
        st = A.accmg_get_stats()
    finally:
        A.accmg_finalize()
    pts = (n - 2) ** 3
    ms_launch = st["ms_body"] / max(st["body_launches"], 1)
    out = {"config": "f2_jacobi3d", "P": P, "n": n, "sweeps": sweeps, "declared": declared,
           "iters_per_s": pts * sweeps / t, "ms_per_loop": t / sweeps * 1e3, **per_loop(st, sweeps),
           "body_GBs": 8 * pts / P / (ms_launch / 1e3) / 1e9}
    out["body_frac_of_measured_hbm"] = out["body_GBs"] / peaks()["hbm_gbs"]
    return out


def deep_cfg(N, sweeps, P, h):
    """§8 row f2 (deep halos): `sweeps` Jacobi sweeps as sweeps/h loops of the deep-halo body —
    one exchange of h halo rows per side per h sweeps, halo rows recomputed redundantly."""
    Ah = gen.jacobi_field(2, N)
    Bh = Ah.copy()
    loops = sweeps // h
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
        for s in range(2):
            WL.jacobi_deep_loop(rA, rB, s, N, h)
        A.accmg_barrier()
        A.accmg_reset_stats()
        t = wall(lambda: [WL.jacobi_deep_loop(rA, rB, s, N, h) for s in range(2, 2 + loops)])
        st = A.accmg_get_stats()
    finally:
        A.accmg_finalize()
    out = {"config": "f2_deep_halo", "P": P, "N": N, "h": h, "sweeps": loops * h,
           "iters_per_s": (N - 2) ** 2 * loops * h / t, "ms_per_sweep": t / (loops * h) * 1e3,
           "exchanges_per_sweep": 1.0 / h, **{k + "_per_sweep": v / h for k, v in per_loop(st, loops).items()}}
    return out


def footprint_cfg(P):
    """§8 row f4 / Fig. 9 (L249-252): device memory per configuration — User (replicas) and
    System (bitmaps, packed buffers, partials, miss buffers) — normalised to the P=1 User total."""
    rows = []
    N = 32768
    for declared in (True, False):
        Ah = gen.jacobi_field(2, N)
        Bh = Ah.copy()
        A.accmg_init(num_partitions=P, device=0)
        try:
            rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
            for s in range(2):
                WL.jacobi_sweep(rA, rB, s, N, declared)
            st = A.accmg_get_stats()
        finally:
            A.accmg_finalize()
        one = 2 * N * N * 4
        rows.append({"config": "f4_footprint", "workload": "c2" if declared else "c5", "P": P,
                     "user_bytes": st["device_bytes_user"], "system_bytes": st["device_bytes_system"],
                     "user_rel_1gpu": st["device_bytes_user"] / one, "system_rel_1gpu": st["device_bytes_system"] / one})
    return rows


def chunk_sweep_cfg(P):
    """§8 row f3 / E7 (L135: "we experimentally choose 1MB"): loop time and inter-partition bytes of
    undeclared writes vs the second-level chunk size, for the paper's protocol (whole chunks +
    bits) and for compacted runs; a sparse writer (every 100th row of 16384^2) and a dense one (C5)."""
    rows = []
    N = 16384
    for body in ("sparse", "dense"):
        for proto in (A.DIRTY_RUNS, A.DIRTY_CHUNKS):
            for cb in (1 << 12, 1 << 14, 1 << 16, 1 << 18, 1 << 20, 1 << 22, 1 << 24):
                src = gen.jacobi_field(7, N)
                dst = src.copy()
                A.accmg_init(num_partitions=P, device=0, profile=1, dirty_chunk_bytes=cb, dirty_protocol=proto)
                try:
                    rs, rd = A.accmg_region_create(src), A.accmg_region_create(dst)
                    def loop(s):
                        if body == "sparse":
                            A.accmg_loop_launch(A.bounds([0], [N]), A.BODY_TEST_SPARSE_WRITE,
                                                [A.access(rs, A.R), A.access(rd, A.W)], A.accmg_args_sparse(N, N, 100))
                        else:
                            WL.jacobi_sweep(rs, rd, s, N, False)
                    loop(0)
                    loop(1)
                    A.accmg_barrier()
                    A.accmg_reset_stats()
                    reps = 5
                    t = wall(lambda: [loop(s) for s in range(2, 2 + reps)])
                    st = A.accmg_get_stats()
                finally:
                    A.accmg_finalize()
                rows.append({"config": "f3_chunk_sweep", "body": body, "P": P,
                             "protocol": "chunks" if proto == A.DIRTY_CHUNKS else "runs", "chunk_bytes": cb,
                             "ms_per_loop": t / reps * 1e3, "bytes_per_loop": st["bytes_interpartition"] / reps,
                             "ms_compact": st["ms_compact"] / reps, "ms_exchange": st["ms_exchange"] / reps})
    return rows


def scatter_cfg(n, P, reps):
    """§8 row f1: irregular writes dst[idx[i]] = src[i] (idx a random permutation) to a distributed
    array; (P-1)/P of the writes miss the writer's window and go through the system buffers."""
    src = gen.jacobi_field(3, 16384, 0, 16384).reshape(-1)[:n].copy()
    idx = gen.permutation(11, n)
    dst = np.zeros(n, np.float32)
    A.accmg_init(num_partitions=P, device=0, profile=1)
    try:
        regs = [A.accmg_region_create(a) for a in (src, idx, dst)]
        WL.scatter_loop(*regs, n, n)
        A.accmg_barrier()
        A.accmg_reset_stats()
        t = wall(lambda: [WL.scatter_loop(*regs, n, n) for _ in range(reps)])
        st = A.accmg_get_stats()
    finally:
        A.accmg_finalize()
    out = {"config": "f1_scatter", "P": P, "n": n, "reps": reps, "iters_per_s": n * reps / t,
           "ms_per_loop": t / reps * 1e3, **per_loop(st, reps),
           "write_misses_per_loop": st["write_misses"] / reps, "bytes_write_miss_per_loop": st["bytes_write_miss"] / reps}
    return out


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--configs", default="c1,c2,c5,c3,c4")
    p.add_argument("--partitions", default="1,2,4,8")
    p.add_argument("--sweeps", type=int, default=100)
    p.add_argument("--c5-sweeps", type=int, default=10)
    p.add_argument("--gemm-n", type=int, default=32768)
    p.add_argument("--gemm-reps", type=int, default=3)
    p.add_argument("--kmeans-n", type=int, default=1 << 28)
    p.add_argument("--kmeans-iters", type=int, default=20)
    p.add_argument("--check", action="store_true", help="k-means closed-form check")
    a = p.parse_args()
    Ps = [int(x) for x in a.partitions.split(",")]
    for cfg in a.configs.split(","):
        for P in Ps:
            try:
                if cfg == "c1":
                    if P in (1, 2):
                        emit(jacobi_cfg("c1", 256, 10, P, True, True))
                elif cfg == "c2":
                    emit(jacobi_cfg("c2", 32768, a.sweeps, P, True, a.check and P == Ps[-1]))
                elif cfg == "c5":
                    emit(jacobi_cfg("c5", 32768, a.c5_sweeps, P, False, a.check and P == Ps[-1]))
                elif cfg == "c3":
                    emit(gemm_cfg(a.gemm_n, P, a.gemm_reps, a.check))
                elif cfg == "f2":
                    emit(jacobi3d_cfg(1024, 20, P))
                elif cfg == "f2u":  # 3-D stencil without declarations: tracked body + compaction + propagation
                    emit(jacobi3d_cfg(1024, 6, P, declared=False))
                elif cfg == "f2deep":
                    for h in (1, 2, 4, 8):
                        emit(deep_cfg(32768, 48, P, h))
                elif cfg == "f3":
                    for row in chunk_sweep_cfg(P):
                        emit(row)
                elif cfg == "f4":
                    for row in footprint_cfg(P):
                        emit(row)
                elif cfg == "f1":
                    emit(scatter_cfg(1 << 26, P, 5))
                elif cfg == "c4":
                    emit(kmeans_cfg(a.kmeans_n, a.kmeans_iters, P, a.check))
                elif cfg == "c4x":  # C4 through exact mode (arbitrary-data path: scalar loop + windows)
                    emit(kmeans_cfg(a.kmeans_n, a.kmeans_iters, P, a.check, exact=True))
            except Exception as e:  # report and continue with the next config
                emit({"config": cfg, "P": P, "error": repr(e)})


if __name__ == "__main__":
    main()
