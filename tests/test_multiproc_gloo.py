"""The N>1 (one process per GPU) host logic on CPU: world_size-2 `gloo` process group, the library
in dry-run mode (device = -1: planning and accounting, no CUDA). Every rank must hold the same
validity table after every loop (the collective-call contract), and the per-rank byte counters
must sum to the oracle model's whole-job totals (pulls counted by the receiving rank)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, V, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    A.accmg_init(num_partitions=world * V, world_size=world, rank=rank, device=-1, halo_mode=A.HALO_PULL)
    N, S = 64, 5
    hA = np.zeros((N, N), np.float32)
    hB = np.zeros((N, N), np.float32)
    rA, rB = A.accmg_region_create(hA), A.accmg_region_create(hB)
    tables, per = [], []
    prev = A.accmg_get_stats()
    for s in range(S):
        WL.jacobi_sweep(rA, rB, s, N, True)
        cur = A.accmg_get_stats()
        per.append({k: cur[k] - prev[k] for k in ("bytes_declared", "bytes_h2d", "bytes_remote")})
        prev = cur
        tables.append([[A.accmg_debug_valid(r, g) for g in range(world * V)] for r in (rA, rB)])
    n, d, k = 1000, 16, 8
    regs = [A.accmg_region_create(a) for a in (np.zeros((n, d), np.float32), np.zeros((k, d), np.float32),
                                                np.zeros(n, np.int32), np.zeros((k, d), np.int64),
                                                np.zeros(k, np.int64))]
    WL.kmeans_loops(*regs, n, d, k)
    red = A.accmg_get_stats()["bytes_reduce"]
    A.accmg_finalize()
    allt = [None] * world
    dist.all_gather_object(allt, (tables, per, red))
    if rank == 0:
        q.put(allt)
    dist.destroy_process_group()


@pytest.mark.parametrize("V", [1, 2])
def test_two_ranks_agree_and_sum_to_model(V):
    from oracle import model as M
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_worker, args=(world, _free_port(), V, q), nprocs=world, join=True, start_method="spawn")
    allt = q.get(timeout=60)
    # identical validity tables on both ranks after every loop
    assert allt[0][0] == allt[1][0]
    # per-loop byte sums over ranks == the oracle model's whole-job numbers
    N, S, P = 64, 5, world * V
    mdl = M.Model(P)
    mA, mB = mdl.region(N * N, 4), mdl.region(N * N, 4)
    for s in range(S):
        src, dst = (mA, mB) if s % 2 == 0 else (mB, mA)
        exp = mdl.loop(1, N - 1, [(src, M.R, 1, N, N, N), (dst, M.W, 1, N, 0, 0)])
        got = {k: sum(allt[r][1][s][k] for r in range(world)) for k in ("bytes_declared", "bytes_h2d")}
        assert got["bytes_declared"] == exp["declared"]
        assert got["bytes_h2d"] == exp["h2d"]
        if s >= 2:   # steady state: the halo rows at the rank boundary cross processes
            assert sum(allt[r][1][s]["bytes_remote"] for r in range(world)) == 2 * 4 * N
    assert sum(a[2] for a in allt) == 2 * (P - 1) * (8 * 16 + 8) * 8
