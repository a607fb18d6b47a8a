#!/usr/bin/env python3
"""Benchmark of the hot path (BASELINE.json configs[1], "C2"): one offloaded parallel loop =
one 5-point Jacobi sweep of a 32768 x 32768 fp32 field, row-block partitioned over the GPUs
with declared halo exchange (localaccess, L87). A step = one accmg_loop_launch (partition ->
halo pull -> body -> coherence bookkeeping).

  python bench.py [--gpus N --steps K --warmup W]               # N>1 under torchrun
  python bench.py --impl reference ...                          # the CPU oracle as reference arm

Prints ONE JSON line on rank 0. Inputs (2 x 4 GiB) are larger than the 126 MB L2, so no flush is
needed between steps. Timing: CUDA events on the library stream, barrier + synchronize on both
sides, max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "loop iters/sec at 1/2/4/8 B200 + % HBM roofline; inter-GPU bytes/loop"
UNIT = "loop iters/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=200)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="accmg", choices=["accmg", "reference"])
    p.add_argument("--size", type=int, default=32768, help="field size N (C2: 32768)")
    p.add_argument("--undeclared", action="store_true", help="C5: no access directives (dirty-bit path)")
    p.add_argument("--e2e-steps", type=int, default=3, help="end-to-end steps (copy-in, 100 sweeps, copy-out)")
    p.add_argument("--e2e-sweeps", type=int, default=100)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    return p.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---- clocks during the timed region -------------------------------------------------------------
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self.stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.01)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0}, "fallback"


def ncu_traffic(kernel_key: str):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f).get(kernel_key)
    except Exception:
        return None


# ---- CPU oracle legs -----------------------------------------------------------------------------
def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def oracle_jacobi_rate(n: int, target_s: float = 10.0, steps: int = 0, warmup: int = 0, threads: int = 0,
                       max_rows: int = 8190):
    """The oracle (oracle/oracle.c, as it stands) on a bounded sample of the C2 workload: full-width
    row bands of the n x n field, repeated sweeps for ~target_s seconds (or, with steps > 0, warmup
    untimed sweeps then exactly `steps` timed sweeps: one step = one sweep of the band), on all
    host cores (threads = 0) or on `threads` of them."""
    import gen
    import oracle
    cores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    if threads:
        cores = min(threads, cores)
    rows = min(max_rows, n - 2)  # 8192 x n band at C2: 1 GiB per array, far larger than any host cache
    band = gen.jacobi_field(2, n, 0, rows + 2)  # a band of the real field (rows 0..rows+1)
    band = np.ascontiguousarray(band)
    # the oracle sweeps a square array; use a (rows+2) x n band embedded as its own field:
    # its interior rows are exactly C2 rows 1..rows (same arithmetic per point)
    out = band.copy()
    for _ in range(warmup):
        oracle.jacobi_sweep_rect(band, out, nthreads=cores)
    t0 = time.perf_counter()
    reps = 0
    while True:
        oracle.jacobi_sweep_rect(band, out, nthreads=cores)
        reps += 1
        if (steps > 0 and reps >= steps) or (steps <= 0 and time.perf_counter() - t0 > target_s):
            break
    dt = time.perf_counter() - t0
    upd = reps * rows * (n - 2)
    return upd / dt, cores, f"{reps} sweeps of a {rows + 2}x{n} band of the C2 field (oracle.jacobi_sweep_rect, {cores} OpenMP threads)"


# ---- the accmg arm -------------------------------------------------------------------------------
def run_accmg(args):
    import torch
    ws, rank, local = dist_env()
    if ws != args.gpus:
        if args.gpus > 1:
            sys.exit(f"--gpus {args.gpus} needs torchrun with {args.gpus} processes")
    dev = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(dev)
    dist = None
    if ws > 1:
        # host-side plumbing only (barriers, max-over-ranks, id broadcast); the data path is the
        # library's own P2P transport over NVLink
        import torch.distributed as dist
        dist.init_process_group("gloo")
    import gen
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL

    N = args.size
    declared = not args.undeclared
    uid = None
    if ws > 1:
        obj = [A.accmg_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    A.accmg_init(num_partitions=ws, world_size=ws, rank=rank, device=dev, profile=1, nccl_unique_id=uid)
    stream = torch.cuda.ExternalStream(A.accmg_stream(), device=dev)

    # host arrays: full extent (virtual), only this rank's rows (+halo) are generated and read
    a, b = A.accmg_chunk(1, N - 1, ws, rank)
    r0, r1 = (a - 1, b + 1) if declared else (0, N)
    Ah = np.empty((N, N), dtype=np.float32)
    Bh = np.empty((N, N), dtype=np.float32)
    gen.jacobi_field(2, N, r0, r1, out=Ah[r0:r1])
    Bh[r0:r1] = Ah[r0:r1]
    rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)

    def barrier():
        stream.synchronize()
        torch.cuda.synchronize()
        if dist:
            dist.barrier()

    for s in range(args.warmup):
        WL.jacobi_sweep(rA, rB, s, N, declared)
    barrier()
    # timed region: no per-phase events between the loops (consecutive bodies overlap their launch
    # with the previous body's tail: programmatic dependent launch)
    A.accmg_set_profile(False)
    A.accmg_reset_stats()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) as clk:
        barrier()
        e0.record(stream)
        for s in range(args.warmup, args.warmup + args.steps):
            WL.jacobi_sweep(rA, rB, s, N, declared)
        e1.record(stream)
        barrier()
    ms = e0.elapsed_time(e1)
    st = A.accmg_get_stats()
    # the body kernel's own duration: the same loops again, bracketed per body by the library's
    # CUDA events on its stream (profile mode)
    A.accmg_set_profile(True)
    A.accmg_reset_stats()
    for s in range(args.warmup + args.steps, args.warmup + 2 * args.steps):
        WL.jacobi_sweep(rA, rB, s, N, declared)
    barrier()
    stp = A.accmg_get_stats()
    t = torch.tensor([ms], dtype=torch.float64)
    tb = torch.tensor([st["bytes_interpartition"], st["kernel_launches"], st["bytes_link"], st["bytes_link_remote"]],
                      dtype=torch.float64)
    if dist:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(tb, op=dist.ReduceOp.SUM)  # byte counters are per process
    ms = float(t.item())
    iters = (N - 2) ** 2 * args.steps                  # loop-body iterations of the whole job
    value = iters / (ms / 1e3)

    # roofline of the dominant kernel (the Jacobi body): algorithmic 8 B per point update
    peaks, peak_src = measured_peaks()
    # the body's launch duration in the timed region: with one body launch per step (one partition
    # per process) the step time itself bounds it from above (it includes the launch gaps); else the
    # profiled pass's per-launch events
    body_ms_prof = stp["ms_body"] / max(stp["body_launches"], 1)
    one_body = st["body_launches"] == args.steps
    body_ms = min(ms / args.steps, body_ms_prof) if one_body else body_ms_prof
    rows_g = b - a
    alg_bytes = 8 * rows_g * (N - 2)
    achieved = alg_bytes / (body_ms / 1e3) / 1e9
    # the committed ncu capture is of the N=32768, one-partition launch; other shapes report none
    traffic = ncu_traffic("jacobi2d_tma") if (N == 32768 and ws == 1) else None
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
            "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": traffic,
            "peak_source": peak_src, "kernel": "jacobi2d_tma_k (TMA-staged tiles)", "algorithmic_bytes_per_launch": alg_bytes,
            "avg_launch_ms": round(body_ms, 4),
            "avg_launch_method": ("timed region: CUDA events around the loops on the library stream, one body "
                                  "launch per loop (step time / steps, gaps included)" if one_body and
                                  body_ms == ms / args.steps else
                                  "CUDA events around each body launch on the library stream (profiled pass of the "
                                  "same number of loops)"),
            "avg_launch_ms_profiled_pass": round(body_ms_prof, 4),
            # also against the 8 TB/s HBM3e specification the north star quotes
            "frac_of_spec_8000GBs": round(achieved / 8000.0, 4)}
    bytes_loop = float(tb[0]) / max(st["loops"], 1)
    link_loop, link_remote_loop = float(tb[2]) / max(st["loops"], 1), float(tb[3]) / max(st["loops"], 1)
    launches = int(tb[1])

    A.accmg_region_destroy(rA)
    A.accmg_region_destroy(rB)
    del Ah, Bh

    # end-to-end through the public API: pinned host buffers, copy-in, 100 sweeps, copy-out
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, A, WL, torch, stream, dist, ws, rank, dev, declared)

    out = None
    if rank == 0:
        out = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
               "warmup": args.warmup, "ms_per_step": round(ms / args.steps, 5), "higher_is_better": True,
               "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
               "config": {"workload": f"C2: 2D 5-point Jacobi {N}x{N} fp32, row-block partition, "
                                      + ("declared halo h=1" if declared else "undeclared (dirty-bit tracking)"),
                          "n": N, "partitions": ws, "sweeps_per_step": 1,
                          "l2_flush": "not needed: 2 x 4 GiB working set >> 126 MB L2",
                          "parallelism": f"row-block x{ws}"},
               "roofline": roof,
               "inter_gpu_bytes_per_loop": bytes_loop,
               "link_bytes_per_loop": link_loop,
               "link_remote_bytes_per_loop": link_remote_loop,
               "gpu_launches": launches,
               "clocks": clk.summary()}
        if e2e:
            out["e2e"] = e2e
    A.accmg_finalize()
    return out


def gpu_numa_cpus(dev: int):
    """CPUs of the NUMA node the GPU hangs off (sysfs), or None."""
    try:
        import pynvml
        pynvml.nvmlInit()
        bus = pynvml.nvmlDeviceGetPciInfo(pynvml.nvmlDeviceGetHandleByIndex(dev)).busId
        bus = bus.decode() if isinstance(bus, bytes) else bus
        bus = bus.lower()[-12:]  # domain:bus:device.function, 0000:xx:yy.z
        node = int(open(f"/sys/bus/pci/devices/{bus}/numa_node").read())
        if node < 0:
            return None
        cpus = set()
        for part in open(f"/sys/devices/system/node/node{node}/cpulist").read().strip().split(","):
            lo, _, hi = part.partition("-")
            cpus.update(range(int(lo), int(hi or lo) + 1))
        return cpus & os.sched_getaffinity(0) or None
    except Exception:
        return None


def run_e2e(args, A, WL, torch, stream, dist, ws, rank, local, declared):
    """End to end through the C ABI: per step region_create + copy-in (the first loop's data loader
    pulls this rank's windows from pinned host memory) + the sweeps + sync_to_host_owned of the result
    + region_destroy, host wall clock, max over ranks. Host buffers are pinned (cudaHostAlloc through
    torch) and allocated and generated by threads of the GPU's NUMA node."""
    N = args.size
    a, b = A.accmg_chunk(1, N - 1, ws, rank)
    r0, r1 = (a - 1, b + 1) if declared else (0, N)
    old_aff = os.sched_getaffinity(0)
    near = gpu_numa_cpus(local)
    if near:
        os.sched_setaffinity(0, near)
    try:
        import gen
        pin = [torch.empty(((r1 - r0), N), dtype=torch.float32, pin_memory=True) for _ in range(2)]
        pa, pb = pin[0].numpy(), pin[1].numpy()
        gen.jacobi_field(2, N, r0, r1, out=pa)
        pb[...] = pa
        A0 = pa.copy()
        # the rank's rows of the region arrays live in the pinned buffers: numpy views with the
        # full-extent geometry, the region's host pointer is the (virtual) element 0
        base = pa.ctypes.data - r0 * N * 4
        Ah = np.ndarray((N, N), dtype=np.float32, buffer=(ctypes_buf(base, N * N * 4)))
        Bh = np.ndarray((N, N), dtype=np.float32, buffer=(ctypes_buf(pb.ctypes.data - r0 * N * 4, N * N * 4)))
    finally:
        os.sched_setaffinity(0, old_aff)
    times, ph, h2d, d2h = [], [], 0, 0
    for step in range(args.e2e_steps + 1):  # first is warm-up
        pa[...] = A0
        pb[...] = A0
        stream.synchronize()
        if dist:
            dist.barrier()
        A.accmg_reset_stats()
        t0 = time.perf_counter()
        rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
        WL.jacobi_sweep(rA, rB, 0, N, declared)   # copy-in (data loader) + sweep 1
        A.accmg_barrier()
        t1 = time.perf_counter()
        for s in range(1, args.e2e_sweeps):
            WL.jacobi_sweep(rA, rB, s, N, declared)
        A.accmg_barrier()
        t2 = time.perf_counter()
        A.accmg_sync_to_host_owned(rA)            # the result (even sweep count: A)
        t3 = time.perf_counter()
        st = A.accmg_get_stats()
        A.accmg_region_destroy(rA)
        A.accmg_region_destroy(rB)
        dt = time.perf_counter() - t0
        tt = torch.tensor([dt], dtype=torch.float64)
        if dist:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        if step > 0:
            times.append(float(tt.item()))
            sweep = (t2 - t1) / max(args.e2e_sweeps - 1, 1)
            ph.append((t1 - t0 - sweep, t2 - t1 + sweep, t3 - t2, time.perf_counter() - t3))
            h2d, d2h = st["bytes_h2d"], st["bytes_d2h"]
    t = float(np.median(times))
    cin, comp, cout, rest = (float(np.median([p[i] for p in ph])) for i in range(4))
    del Ah, Bh, pa, pb, pin
    return {"value": round((N - 2) ** 2 * args.e2e_sweeps / t, 1), "unit": UNIT, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "sweeps_per_step": args.e2e_sweeps, "seconds_per_step": round(t, 4),
            "phases_s": {"copy_in": round(cin, 4), "sweeps": round(comp, 4), "copy_out": round(cout, 4),
                         "stats_destroy": round(rest, 4)},
            "h2d_GBs": round(h2d / cin / 1e9, 2) if cin > 0 else None,
            "d2h_GBs": round(d2h / cout / 1e9, 2) if cout > 0 else None,
            "host_numa_bound": bool(near),
            "note": "host wall clock per step: region_create + copy-in from pinned host (data loader of the "
                    "first loop) + sweeps + sync_to_host_owned of the result + region_destroy, max over ranks; "
                    "per-rank bytes; copy_in = first loop minus one sweep"}


def ctypes_buf(addr: int, nbytes: int):
    import ctypes
    return (ctypes.c_uint8 * nbytes).from_address(addr)


def free_port() -> int:
    import socket
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def self_launch(n: int) -> int:
    """`python bench.py --gpus N` without torchrun: re-run this script as N ranks (one process per
    GPU, rank r on device r % device_count) through torch.distributed.run on 127.0.0.1. Rank 0's
    JSON line is the only stdout line; the exit code is torchrun's."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    args = parse()
    ws, rank, local = dist_env()
    if args.impl == "accmg" and args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(self_launch(args.gpus))
    if args.impl == "reference":
        if rank != 0:
            return
        rate, cores, sample = oracle_jacobi_rate(args.size, steps=max(args.steps, 1), warmup=args.warmup)
        line = {"impl": "reference", "metric": METRIC, "value": round(rate, 1), "unit": UNIT, "n_gpus": args.gpus,
                "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "vs_baseline": None,
                "dtype": "f32", "data": "synthetic",
                # the accmg arm's workload; the bounded host sample is described in cpu_baseline.sample
                "config": {"workload": f"C2: 2D 5-point Jacobi {args.size}x{args.size} fp32, row-block partition, "
                                       + ("undeclared (dirty-bit tracking)" if args.undeclared else "declared halo h=1"),
                           "n": args.size, "partitions": 1, "sweeps_per_step": 1, "parallelism": "oracle on host cores"},
                "cpu_baseline": {"value": round(rate, 1), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                                 "cpu_model": cpu_model()},
                "e2e": {"value": round(rate, 1), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return
    out = run_accmg(args)
    if rank == 0:
        if not args.no_cpu_baseline and ws == 1:  # the host baseline is taken at N = 1 only
            rate, cores, sample = oracle_jacobi_rate(args.size, target_s=10.0)
            rate1, _, sample1 = oracle_jacobi_rate(args.size, target_s=4.0, threads=1, max_rows=1022)
            out["cpu_baseline"] = {"value": round(rate, 1), "unit": UNIT, "cores": cores, "kind": "oracle",
                                   "sample": sample, "cpu_model": cpu_model(),
                                   "single_core": {"value": round(rate1, 1), "unit": UNIT, "cores": 1,
                                                   "sample": sample1}}
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
