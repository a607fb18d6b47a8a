"""One process per GPU (SPMD) through the C ABI: two processes share the one B200 available
in-round (each its own CUDA context), exchanging through CUDA IPC mappings (P2P mode) and a
device-side flag barrier — the same code path as one process per GPU on an NVSwitch box. Results
must equal the oracle bit for bit on every rank, and the per-rank byte counters must sum to the
single-process totals."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _device_count():
    import torch
    return torch.cuda.device_count()


def _launch(world, V, work, tmp_path, mode=0, devices=None, multicast=0):
    """One process per rank; rank r runs on devices[r] (default r % device_count: one GPU per rank
    on a multi-GPU box, all ranks on the one GPU otherwise)."""
    uid = os.urandom(128).hex()
    nd = _device_count()
    devices = devices or [r % nd for r in range(world)]
    procs = [subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "mp_worker.py"), str(r), str(world), str(V),
                               uid, work, str(tmp_path), str(mode), str(devices[r]), str(multicast)], cwd=ROOT)
             for r in range(world)]
    for p in procs:
        assert p.wait(timeout=600) == 0
    stats = [json.load(open(tmp_path / f"rank{r}_stats.json")) for r in range(world)]
    return stats


@pytest.mark.parametrize("work,V", [("jacobi_decl", 1), ("jacobi_decl", 2), ("jacobi_undecl", 1), ("jacobi_undecl", 2)])
def test_jacobi_two_processes(tmp_path, work, V):
    N, S = 300, 6
    A0 = gen.jacobi_field(5, N)
    oA, oB = A0.copy(), A0.copy()
    oracle.jacobi_run(oA, oB, S)
    stats = _launch(2, V, work, tmp_path)
    for r in range(2):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_A.npy"), oA)
        assert np.array_equal(np.load(tmp_path / f"rank{r}_B.npy"), oB)
    P = 2 * V
    tot = sum(s["bytes_interpartition"] for s in stats)
    if work == "jacobi_decl":  # boundary rows pushed by the bodies (the last loop's push is unused)
        assert sum(s["bytes_declared"] for s in stats) == S * 2 * (P - 1) * 4 * N
    else:
        assert tot == S * (P - 1) * (16 * P + 16 * (N - 2) + 4 * (N - 2) ** 2)
    assert sum(s["bytes_remote"] for s in stats) > 0


@pytest.mark.parametrize("world,V", [(2, 2), (3, 1)])
def test_kmeans_multi_process(tmp_path, world, V):
    """Tensor-core assignment on each rank's points, reductiontoarray partials summed across the
    ranks through the IPC mappings; centroids and assignments bit-exact on every rank."""
    x = gen.kmeans_points(5, 20000, 16, 32, gen.KM_OVERLAP)
    ocen, omem = oracle.kmeans_run(x, 32, 5)
    stats = _launch(world, V, "kmeans", tmp_path)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_cen.npy"), ocen)
        assert np.array_equal(np.load(tmp_path / f"rank{r}_mem.npy"), omem)
    P = world * V
    # each rank books its integer share of every all-reduce (2 regions x 5 iterations)
    assert abs(sum(s["bytes_reduce"] for s in stats) - 5 * 2 * (P - 1) * (32 * 16 + 32) * 8) < world * 5 * 2
    # link bytes: every process reads the P-1 other partials of each reduction over the IPC
    # mappings (P(P-1) S in total with one partition per process); the update loop's writes to the
    # replicated centroids / sums / counts are pushed to the P-1 other replicas (payload only); the
    # final non-owned sync_to_host of member pulls what each process does not hold
    S, k, d, n, iters = (32 * 16 + 32) * 8, 32, 16, 20000, 5
    upd = k * d * 4 + (k * d + k) * 8
    exp = world * iters * (P - 1) * S + iters * (P - 1) * upd + (world - 1) * n * 4
    assert sum(s["bytes_link"] for s in stats) == exp
    exp_remote = world * iters * (P - V) * S + iters * (P - V) * upd + (world - 1) * n * 4
    assert sum(s["bytes_link_remote"] for s in stats) == exp_remote


def test_scatter_two_processes(tmp_path):
    """Write misses completed directly in a peer process's replica through its IPC mapping."""
    n = 50000
    src = gen.jacobi_field(3, 317, 0, 317).reshape(-1)[:n].copy()
    idx = gen.permutation(11, n)
    exp = np.zeros(n, np.float32)
    miss = oracle.scatter(src, idx, exp, P=4)
    stats = _launch(2, 2, "scatter", tmp_path)
    for r in range(2):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_dst.npy"), exp)
    assert sum(s["write_misses"] for s in stats) == int(miss.sum())


@pytest.mark.parametrize("world,V", [(2, 2), (3, 1), (3, 2)])
def test_masked_writes_multi_process(tmp_path, world, V):
    """Irregular undeclared writes (isolated bits, runs across tiles and chunks) across processes:
    each rank's compaction pass pushes its dirty elements into the peer's replicas through the IPC
    mappings; every rank ends bit-exact. (NCCL cannot put two ranks on one GPU; its packed-buffer
    path is covered in-process by the XCHG_NCCL_ALL tests.)"""
    n = (1 << 20) + 4321
    src = (gen.u_fill(21, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
    exp = np.full(n, -1.0, dtype=np.float32)
    for seed, dens, run in ((22, 0.5, 1), (23, 0.3, 70001), (24, 0.9, 40)):
        oracle.masked_write(src, gen.write_mask(seed, n, dens, run), exp)
    _launch(world, V, "masked", tmp_path)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_out.npy"), exp)


def test_undeclared_first_loop_copy_in_before_peer_pushes(tmp_path):
    """Regression: in the first undeclared loop every rank copies the host array into its replica
    while its peers, after their bodies, push their dirty rows into it. Without a barrier between
    the loader's copies and the bodies, a slow rank's copy-in could overwrite a fast peer's pushed
    rows (it did in ~1 of 8 three-rank runs on one GPU: wrong values around the partition
    boundaries, identical on every rank). Eight repetitions, each bit-exact."""
    N, S = 300, 6
    A0 = gen.jacobi_field(5, N)
    oA, oB = A0.copy(), A0.copy()
    oracle.jacobi_run(oA, oB, S)
    for rep in range(8):
        d = tmp_path / f"rep{rep}"
        d.mkdir()
        _launch(3, 1, "jacobi_undecl", d)
        for r in range(3):
            assert np.array_equal(np.load(d / f"rank{r}_A.npy"), oA), (rep, r)
            assert np.array_equal(np.load(d / f"rank{r}_B.npy"), oB), (rep, r)


@pytest.mark.parametrize("work", ["jacobi_decl", "jacobi_undecl"])
def test_jacobi_three_processes(tmp_path, work):
    """Three ranks (partitions 0-2 in three CUDA contexts): the middle rank pushes halos / dirty
    elements to two IPC-mapped peers per loop; every rank bit-exact."""
    N, S = 300, 6  # tests/mp_worker.py runs 6 sweeps of the 300 x 300 field
    A0 = gen.jacobi_field(5, N)
    oA, oB = A0.copy(), A0.copy()
    oracle.jacobi_run(oA, oB, S)
    stats = _launch(3, 1, work, tmp_path)
    for r in range(3):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_A.npy"), oA)
        assert np.array_equal(np.load(tmp_path / f"rank{r}_B.npy"), oB)
    if work == "jacobi_undecl":
        P = 3
        assert sum(s["bytes_interpartition"] for s in stats) == S * (P - 1) * (16 * P + 16 * (N - 2) + 4 * (N - 2) ** 2)


@pytest.mark.parametrize("world,V", [(2, 2), (3, 1)])
def test_kmeans_exact_multi_process(tmp_path, world, V):
    """Exact mode (arbitrary real-valued points, reading KM-X): the nine-window partials of every
    rank are merged across the processes; centroids and assignments bit-exact on every rank."""
    x = gen.kmeans_points_real(46, 12007, 34, 19)
    ocen, omem = oracle.kmeans_run_exact(x, 19, 3)
    stats = _launch(world, V, "kmeans_exact", tmp_path)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_cen.npy"), ocen)
        assert np.array_equal(np.load(tmp_path / f"rank{r}_mem.npy"), omem)
    P = world * V
    assert abs(sum(s["bytes_reduce"] for s in stats) - 3 * 2 * (P - 1) * (19 * 34 * 9 + 19) * 8) < world * 3 * 2


@pytest.mark.parametrize("work", ["jacobi_decl", "jacobi_undecl", "kmeans", "masked"])
def test_two_physical_gpus(tmp_path, work):
    """Ranks 0 and 1 on devices 0 and 1: replicas mapped across GPUs through CUDA IPC, halo rows
    posted into the peer's HBM over NVLink by the Jacobi body, dirty elements pushed by the
    compaction pass, reduction partials read over NVLink, and the flag barrier across devices.
    Every rank bit-exact against the oracle."""
    if _device_count() < 2:
        pytest.skip(f"needs 2 physical GPUs, this box has {_device_count()} (the one-GPU runs above cover the same code "
                    "path with both ranks on one device)")
    _launch(2, 1, work, tmp_path, devices=[0, 1])
    if work.startswith("jacobi"):
        N, S = 300, 6
        A0 = gen.jacobi_field(5, N)
        oA, oB = A0.copy(), A0.copy()
        oracle.jacobi_run(oA, oB, S)
        exp = {"A": oA, "B": oB}
    elif work == "kmeans":
        x = gen.kmeans_points(5, 20000, 16, 32, gen.KM_OVERLAP)
        ocen, omem = oracle.kmeans_run(x, 32, 5)
        exp = {"cen": ocen, "mem": omem}
    else:
        n = (1 << 20) + 4321
        src = (gen.u_fill(21, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
        out = np.full(n, -1.0, dtype=np.float32)
        for seed, dens, run in ((22, 0.5, 1), (23, 0.3, 70001), (24, 0.9, 40)):
            oracle.masked_write(src, gen.write_mask(seed, n, dens, run), out)
        exp = {"out": out}
    for r in range(2):
        for k, v in exp.items():
            assert np.array_equal(np.load(tmp_path / f"rank{r}_{k}.npy"), v), (r, k)


@pytest.mark.parametrize("world,V", [(2, 1), (3, 2)])
def test_sync_to_host_right_after_loops(tmp_path, world, V):
    """A 2048^2 declared Jacobi run whose non-owned sync_to_host follows the last loop directly (no
    stats call to synchronise the stream): the replica hulls grow to the full extent there, so the
    hull copies and the previous loop's pushes must complete before the new replicas are published."""
    N, S = 2048, 4
    A0 = gen.jacobi_field(6, N)
    oA, oB = A0.copy(), A0.copy()
    oracle.jacobi_run(oA, oB, S)
    _launch(world, V, "jacobi_decl_sync", tmp_path)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"rank{r}_A.npy"), oA)
        assert np.array_equal(np.load(tmp_path / f"rank{r}_B.npy"), oB)


def _expect(work):
    if work.startswith("jacobi"):
        N, S = 300, 6
        A0 = gen.jacobi_field(5, N)
        oA, oB = A0.copy(), A0.copy()
        oracle.jacobi_run(oA, oB, S)
        return {"A": oA, "B": oB}
    n = (1 << 20) + 4321
    src = (gen.u_fill(21, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
    out = np.full(n, -1.0, dtype=np.float32)
    for seed, dens, run in ((22, 0.5, 1), (23, 0.3, 70001), (24, 0.9, 40)):
        oracle.masked_write(src, gen.write_mask(seed, n, dens, run), out)
    return {"out": out}


@pytest.mark.parametrize("work", ["jacobi_undecl", "masked"])
def test_vmm_replicas_shared_through_descriptors(tmp_path, work):
    """§8 f3 plumbing without the switch (ACCMG_MC_VMM): replicas of arrays written without a
    declared pattern are driver-VMM allocations, exported as file descriptors, passed between the
    processes over Unix sockets and mapped by every peer; the compaction pass pushes the dirty
    elements into them. Two processes, bit-exact on both."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    stats = _launch(2, 1, work, tmp_path, multicast=A.MC_VMM)
    for r in range(2):
        for k, v in _expect(work).items():
            assert np.array_equal(np.load(tmp_path / f"rank{r}_{k}.npy"), v), (r, k)
    tot = stats if isinstance(stats[0], dict) and "multicast_regions" in stats[0] else [s["total"] for s in stats]
    assert all(s["multicast_regions"] == 0 for s in tot)


@pytest.mark.parametrize("work", ["jacobi_undecl", "masked"])
def test_nvls_multicast_push(tmp_path, work):
    """§8 f3: ACCMG_MC_AUTO — where the node can create an NVLS multicast object over the ranks'
    GPUs, the compaction pass stores every dirty element once through the multicast address
    (multimem.st) into all replicas; elsewhere the same run falls back to unicast pushes. Bit-exact
    either way; the multicast assertions are skipped with the probe's reason when unavailable."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    nd = _device_count()
    ok, why = A.accmg_multicast_probe(min(nd, 2))
    stats = _launch(2, 1, work, tmp_path, multicast=A.MC_AUTO)
    for r in range(2):
        for k, v in _expect(work).items():
            assert np.array_equal(np.load(tmp_path / f"rank{r}_{k}.npy"), v), (r, k)
    tot = stats if "multicast_regions" in stats[0] else [s["total"] for s in stats]
    if not (ok and nd >= 2):
        assert all(s["multicast_regions"] == 0 for s in tot)
        pytest.skip(f"NVLS multicast unavailable here (fell back to unicast pushes, bit-exact): {why or 'one GPU'}")
    assert all(s["multicast_regions"] >= 1 for s in tot)
    assert sum(s["bytes_multicast"] for s in tot) > 0


def test_multicast_probe_reports():
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    ok, why = A.accmg_multicast_probe(1)
    assert isinstance(ok, bool)
    assert ok or why
