"""One rank of a multi-process (one process per GPU) run, used by tests/test_gpu_multiproc.py.

usage: python tests/mp_worker.py RANK WORLD V UID_HEX WORKLOAD OUTDIR [EXCHANGE_MODE [DEVICE [MULTICAST]]]
Runs the workload through the C ABI with world_size = WORLD, num_partitions = WORLD * V, and
saves its host arrays (after sync_to_host) and its stats under OUTDIR/rank<R>_*.npy/.json.
DEVICE defaults to 0; the launching test passes rank % device_count (one process per GPU on a
multi-GPU box, ranks sharing the GPU on a one-GPU box).
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import accmg as A  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import workloads as WL  # noqa: E402


def main():
    rank, world, V = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
    uid = bytes.fromhex(sys.argv[4])
    work, out = sys.argv[5], sys.argv[6]
    mode = int(sys.argv[7]) if len(sys.argv) > 7 else A.XCHG_AUTO
    device = int(sys.argv[8]) if len(sys.argv) > 8 else 0
    mc = int(sys.argv[9]) if len(sys.argv) > 9 else A.MC_OFF
    A.accmg_init(num_partitions=world * V, world_size=world, rank=rank, device=device, nccl_unique_id=uid, multicast=mc,
                 exchange_mode=mode, dirty_chunk_bytes=8192)
    res = {}
    if work in ("jacobi_decl", "jacobi_undecl"):
        N, S = 300, 6
        Ah = gen.jacobi_field(5, N)
        Bh = Ah.copy()
        per = WL.jacobi_run(Ah, Bh, S, declared=(work == "jacobi_decl"), per_loop_stats=True)
        res = {"A": Ah, "B": Bh}
        loops = {k: sum(p[k] for p in per) for k in per[0]}
    elif work == "jacobi_decl_sync":
        # no stats call between the loops and sync_to_host: nothing synchronises the stream before
        # the hull growth of the non-owned copy-out (ensure_alloc ordering)
        N, S = 2048, 4
        Ah = gen.jacobi_field(6, N)
        Bh = Ah.copy()
        WL.jacobi_run(Ah, Bh, S, declared=True)
        res = {"A": Ah, "B": Bh}
    elif work == "kmeans":
        x = gen.kmeans_points(5, 20000, 16, 32, gen.KM_OVERLAP)
        cen, mem = WL.kmeans_run(x, 32, 5)
        res = {"cen": cen, "mem": mem}
    elif work == "kmeans_exact":
        x = gen.kmeans_points_real(46, 12007, 34, 19)
        cen, mem = WL.kmeans_run(x, 19, 3, shift=A.KMEANS_EXACT)
        res = {"cen": cen, "mem": mem}
    if work == "masked":
        n = (1 << 20) + 4321
        src = (gen.u_fill(21, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
        dst = np.full(n, -1.0, dtype=np.float32)
        ri, ro = A.accmg_region_create(src), A.accmg_region_create(dst)
        for seed, dens, run in ((22, 0.5, 1), (23, 0.3, 70001), (24, 0.9, 40)):
            m = gen.write_mask(seed, n, dens, run)
            rm = A.accmg_region_create(m)
            A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_TEST_MASKED_WRITE,
                                [A.access(ri, A.R), A.access(rm, A.R), A.access(ro, A.W)], A.accmg_args_masked(n))
            A.accmg_region_destroy(rm)
        A.accmg_sync_to_host(ro)
        res = {"out": dst}
    if work == "scatter":
        n = 50000
        src = gen.jacobi_field(3, 317, 0, 317).reshape(-1)[:n].copy()
        idx = gen.permutation(11, n)
        dst = np.zeros(n, np.float32)
        regs = [A.accmg_region_create(a) for a in (src, idx, dst)]
        WL.scatter_loop(*regs, n, n)
        A.accmg_sync_to_host(regs[2])
        res = {"dst": dst}
    st = A.accmg_get_stats()
    if work in ("jacobi_decl", "jacobi_undecl"):
        st = {"total": st, **loops}
    A.accmg_finalize()
    for k, v in res.items():
        np.save(os.path.join(out, f"rank{rank}_{k}.npy"), v)
    with open(os.path.join(out, f"rank{rank}_stats.json"), "w") as f:
        json.dump(st, f)


if __name__ == "__main__":
    main()
