"""C-ABI library on the CPU: it loads, exports every entry point of include/accmg.h, and its host
logic (task mapping, window/pull planning, validity table, byte accounting, argument checks) —
run in dry-run mode (device = -1: no CUDA call, no body) — matches the oracle's brute-force
coherence model element by element. No GPU needed."""
import numpy as np
import pytest

import oracle
from oracle import model as M
from paper_conf_icpp_komodamnm13_b200 import accmg as A
from paper_conf_icpp_komodamnm13_b200 import workloads as WL


@pytest.fixture
def dry():
    def start(P, **kw):
        A.accmg_init(num_partitions=P, device=-1, **kw)
    yield start
    try:
        A.accmg_finalize()
    except A.AccmgError:
        pass


def test_exports_every_header_symbol():
    syms = A.header_symbols()
    assert len(syms) >= 19
    for s in syms:
        assert hasattr(A._lib, s), s


def test_chunk_matches_oracle_partition():
    for P in range(1, 10):
        for n in range(0, 40):
            for g in range(P):
                assert A.accmg_chunk(3, 3 + n, P, g) == oracle.partition(3, 3 + n, P, g)


def _intervals(mask):
    m = np.concatenate(([0], mask.astype(np.int8), [0]))
    d = np.diff(m)
    return list(zip(np.flatnonzero(d == 1).tolist(), np.flatnonzero(d == -1).tolist()))


def _compare_valid(regs_c, regs_m, P):
    for rc, rm in zip(regs_c, regs_m):
        for g in range(P):
            assert A.accmg_debug_valid(rc, g) == _intervals(rm.valid[g]), g
        assert A.accmg_debug_valid(rc, -1) == _intervals(rm.host_valid)


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_declared_jacobi_plan_vs_model(dry, P):
    N, S = 40, 5
    dry(P, halo_mode=A.HALO_PULL)   # the paper's data loader: pull before read (the model's semantics)
    hA = np.zeros((N, N), np.float32)
    hB = np.zeros((N, N), np.float32)
    rA, rB = A.accmg_region_create(hA), A.accmg_region_create(hB)
    mdl = M.Model(P)
    mA, mB = mdl.region(N * N, 4), mdl.region(N * N, 4)
    for s in range(S):
        before = A.accmg_get_stats()
        WL.jacobi_sweep(rA, rB, s, N, True)
        after = A.accmg_get_stats()
        src, dst = (mA, mB) if s % 2 == 0 else (mB, mA)
        exp = mdl.loop(1, N - 1, [(src, M.R, 1, N, N, N), (dst, M.W, 1, N, 0, 0)])
        assert after["bytes_declared"] - before["bytes_declared"] == exp["declared"]
        assert after["bytes_h2d"] - before["bytes_h2d"] == exp["h2d"]
        _compare_valid([rA, rB], [mA, mB], P)
    A.accmg_sync_to_host(rA)
    assert A.accmg_get_stats()["bytes_d2h"] == mdl.sync_to_host(mA)
    _compare_valid([rA], [mA], P)


@pytest.mark.parametrize("seed", range(12))
def test_random_windows_plan_vs_model(dry, seed):
    """Random localaccess windows (stride, left, right) over random loop bounds (L87)."""
    rng = np.random.default_rng(seed)
    P = int(rng.integers(1, 7))
    rows, cols = int(rng.integers(4, 30)), int(rng.integers(3, 9))
    dry(P)
    h = [np.zeros(rows * cols, np.float32) for _ in range(2)]
    rc = [A.accmg_region_create(x) for x in h]
    mdl = M.Model(P)
    rm = [mdl.region(rows * cols, 4) for _ in range(2)]
    for it in range(4):
        lo = int(rng.integers(0, 3))
        hi = int(rng.integers(lo, rows + 1))
        s = cols
        l, r = int(rng.integers(0, 3 * cols)), int(rng.integers(0, 3 * cols))
        src, dst = (0, 1) if it % 2 == 0 else (1, 0)
        descs = [A.access(rc[src], A.R, True, s, l, r), A.access(rc[dst], A.W, True, s, 0, 0)]
        args = A.accmg_args_sparse(rows, cols, 1)
        before = A.accmg_get_stats()
        A.accmg_loop_launch(A.bounds([lo], [hi]), A.BODY_TEST_SPARSE_WRITE, descs, args)
        after = A.accmg_get_stats()
        exp = mdl.loop(lo, hi, [(rm[src], M.R, 1, s, l, r), (rm[dst], M.W, 1, s, 0, 0)])
        assert after["bytes_declared"] - before["bytes_declared"] == exp["declared"]
        assert after["bytes_h2d"] - before["bytes_h2d"] == exp["h2d"]
        _compare_valid(rc, rm, P)


def test_c1_worked_example_dry(dry):
    N, P = 256, 2
    dry(P)
    h = [np.zeros((N, N), np.float32) for _ in range(2)]
    per = []
    rA, rB = A.accmg_region_create(h[0]), A.accmg_region_create(h[1])
    prev = A.accmg_get_stats()
    for s in range(10):
        WL.jacobi_sweep(rA, rB, s, N, True)
        cur = A.accmg_get_stats()
        per.append(cur["bytes_declared"] - prev["bytes_declared"])
        prev = cur
    assert per[0] == 0 and all(p == 2048 for p in per[2:])
    # W_0 = [256, 32768) is owned by partition 0 after a write of the B array
    assert A.accmg_debug_valid(rB, 0)[0][1] >= 32768


@pytest.mark.parametrize("P", [2, 3, 8])
def test_halo_push_dry(P):
    """halo_mode AUTO: from the second write of an array on, each writer's boundary rows are pushed
    into the neighbours that read them in the previous loop (predicted from L125), so the steady
    state pulls nothing and moves the same bytes per loop; validity is a superset of the pull-only
    loader's (the pushed rows are valid one loop earlier) and the copy-out is identical."""
    N, S = 40, 7
    X = 2 * (P - 1) * 4 * N
    res = {}
    for mode in (A.HALO_PULL, A.HALO_AUTO):
        A.accmg_init(num_partitions=P, device=-1, halo_mode=mode)
        try:
            h = [np.zeros((N, N), np.float32) for _ in range(2)]
            rA, rB = A.accmg_region_create(h[0]), A.accmg_region_create(h[1])
            per, prev = [], A.accmg_get_stats()
            for s in range(S):
                WL.jacobi_sweep(rA, rB, s, N, True)
                cur = A.accmg_get_stats()
                per.append((cur["bytes_declared"] - prev["bytes_declared"], cur["bytes_h2d"] - prev["bytes_h2d"]))
                prev = cur
            valid = [[A.accmg_debug_valid(r, g) for g in range(P)] for r in (rA, rB)]
            A.accmg_sync_to_host(rA)
            res[mode] = (per, valid, A.accmg_get_stats()["bytes_d2h"])
        finally:
            A.accmg_finalize()
    pull, auto = res[A.HALO_PULL], res[A.HALO_AUTO]
    assert [b for b, _ in pull[0]] == [0] + [X] * (S - 1)
    assert [b for b, _ in auto[0]] == [0, 2 * X] + [X] * (S - 2)       # loop 1 pulls B and pushes A
    assert [h for _, h in auto[0]] == [h for _, h in pull[0]]
    assert auto[2] == pull[2]
    for va, vp in zip(auto[1], pull[1]):
        for ga, gp in zip(va, vp):
            cover = np.zeros(N * N, bool)
            for lo, hi in ga:
                cover[lo:hi] = True
            assert all(cover[lo:hi].all() for lo, hi in gp)


def test_reduce_and_replica_bytes_dry(dry):
    n, d, k, P = 1000, 16, 8, 4
    dry(P)
    x = np.zeros((n, d), np.float32)
    regs = [A.accmg_region_create(a) for a in (x, np.zeros((k, d), np.float32), np.zeros(n, np.int32),
                                                np.zeros((k, d), np.int64), np.zeros(k, np.int64))]
    WL.kmeans_loops(*regs, n, d, k)
    st = A.accmg_get_stats()
    assert st["bytes_reduce"] == 2 * (P - 1) * (k * d + k) * 8
    # x is distributed: each partition loads only its points from the host (L121-123)
    assert st["bytes_h2d"] >= n * d * 4 and st["bytes_h2d"] < 2 * n * d * 4 + P * (k * d * 4 + 2 * (k * d + k) * 8)


def test_argument_errors(dry):
    dry(2)
    N = 16
    h = [np.zeros((N, N), np.float32) for _ in range(2)]
    rA, rB = A.accmg_region_create(h[0]), A.accmg_region_create(h[1])
    args = A.accmg_args_jacobi2d(N, N)
    b = A.bounds([1, 1], [N - 1, N - 1])
    good = WL.jacobi_descs(rA, rB, N, True)
    with pytest.raises(A.AccmgError) as e:
        A.accmg_loop_launch(b, 77, good, args)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:   # wrong mode for the body
        A.accmg_loop_launch(b, A.BODY_JACOBI2D_5PT, [good[0], A.access(rB, A.R, True, N)], args)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:   # stride <= 0
        A.accmg_loop_launch(b, A.BODY_JACOBI2D_5PT, [A.access(rA, A.R, True, 0, 0, 0), good[1]], args)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:   # same region twice
        A.accmg_loop_launch(b, A.BODY_JACOBI2D_5PT, [good[0], A.access(rA, A.W, True, N)], args)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:   # bounds outside the interior
        A.accmg_loop_launch(A.bounds([0, 1], [N - 1, N - 1]), A.BODY_JACOBI2D_5PT, good, args)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:   # overlapping declared writes (owner computes, G14)
        A.accmg_loop_launch(b, A.BODY_JACOBI2D_5PT, [good[0], A.access(rB, A.W, True, N, N, 0)], args)
    assert e.value.code == A.ECONFLICT
    A.accmg_loop_launch(b, A.BODY_JACOBI2D_5PT, good, args)   # still usable (errors are not sticky)


def test_state_errors():
    with pytest.raises(A.AccmgError) as e:
        A.accmg_barrier()
    assert e.value.code == A.ESTATE
    with pytest.raises(A.AccmgError) as e:
        A.accmg_init(num_partitions=3, world_size=2, device=-1)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:
        A.accmg_init(num_partitions=65, device=-1)
    assert e.value.code == A.EUNSUPPORTED
    with pytest.raises(A.AccmgError) as e:
        A.accmg_init(num_partitions=1, device=-1, dirty_chunk_bytes=1000)
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:
        A.accmg_init(num_partitions=1, device=-1, dirty_chunk_bytes=128)   # the header's minimum is 256
    assert e.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as e:
        A.accmg_init(num_partitions=1, device=-1, multicast=7)
    assert e.value.code == A.EINVAL
    A.accmg_init(num_partitions=2, device=-1, multicast=A.MC_AUTO)  # dry run: accepted, nothing to bind
    A.accmg_finalize()


def test_scatter_requires_declared_dst(dry):
    dry(2)
    n = 64
    regs = [A.accmg_region_create(a) for a in (np.zeros(n, np.float32), np.zeros(n, np.int32), np.zeros(n, np.float32))]
    with pytest.raises(A.AccmgError) as e:
        A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_SCATTER,
                            [A.access(regs[0], A.R, True, 1), A.access(regs[1], A.R, True, 1), A.access(regs[2], A.W)],
                            A.accmg_args_scatter(n, n))
    assert e.value.code == A.EUNSUPPORTED
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    WL.scatter_loop(*regs, n, n)   # declared: accepted (dry run: planning only)


@pytest.mark.parametrize("P,h", [(2, 2), (4, 3), (8, 8)])
def test_deep_halo_plan_vs_model(dry, P, h):
    """Deep-halo loops (§8 f2): the window of h rows per side, planned as the model plans it."""
    N = 48
    dry(P)
    hA, hB = np.zeros((N, N), np.float32), np.zeros((N, N), np.float32)
    rA, rB = A.accmg_region_create(hA), A.accmg_region_create(hB)
    mdl = M.Model(P)
    mA, mB = mdl.region(N * N, 4), mdl.region(N * N, 4)
    for s in range(4):
        before = A.accmg_get_stats()
        WL.jacobi_deep_loop(rA, rB, s, N, h)
        after = A.accmg_get_stats()
        src, dst = (mA, mB) if s % 2 == 0 else (mB, mA)
        exp = mdl.loop(1, N - 1, [(src, M.R, 1, N, h * N, h * N), (dst, M.W, 1, N, 0, 0)])
        assert after["bytes_declared"] - before["bytes_declared"] == exp["declared"]
        assert after["bytes_h2d"] - before["bytes_h2d"] == exp["h2d"]
        _compare_valid([rA, rB], [mA, mB], P)
    with pytest.raises(A.AccmgError) as e:
        A.accmg_loop_launch(A.bounds([1, 1], [N - 1, N - 1]), A.BODY_JACOBI2D_DEEP,
                            WL.jacobi_deep_descs(rA, rB, N, h), A.accmg_args_jacobi2d_deep(N, N, 0))
    assert e.value.code == A.EINVAL


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_kmeans_assign_reduction_plan_vs_model(dry, P):
    """The k-means assignment loop (reductiontoarray destinations, L89-91 / L112): byte counters and
    validity after each loop match the model's REDUCE_SUM branch, and the reduction bytes equal
    the closed form of reading W8 — 2 (P - 1) x (sums + counts bytes) per loop."""
    n, d, k = 1000, 16, 37
    dry(P)
    hx, hc = np.zeros((n, d), np.float32), np.zeros((k, d), np.float32)
    hm, hs, hn = np.zeros(n, np.int32), np.zeros((k, d), np.int64), np.zeros(k, np.int64)
    rx, rc, rm, rs, rn = (A.accmg_region_create(a) for a in (hx, hc, hm, hs, hn))
    mdl = M.Model(P)
    mx, mc, mm = mdl.region(n * d, 4), mdl.region(k * d, 4), mdl.region(n, 4)
    ms, mn = mdl.region(k * d, 8), mdl.region(k, 8)
    for _ in range(2):
        before = A.accmg_get_stats()
        A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_KMEANS_ASSIGN,
                            [A.access(rx, A.R, True, d, 0, 0), A.access(rc, A.R), A.access(rm, A.W, True, 1, 0, 0),
                             A.access(rs, A.REDUCE_SUM), A.access(rn, A.REDUCE_SUM)], A.accmg_args_kmeans(n, d, k, 8))
        after = A.accmg_get_stats()
        exp = mdl.loop(0, n, [(mx, M.R, 1, d, 0, 0), (mc, M.R, 0, 0, 0, 0), (mm, M.W, 1, 1, 0, 0),
                              (ms, M.REDUCE_SUM, 0, 0, 0, 0), (mn, M.REDUCE_SUM, 0, 0, 0, 0)])
        assert exp["reduce"] == 2 * (P - 1) * (k * d * 8 + k * 8)
        for key in ("reduce", "declared", "h2d", "interpartition"):
            assert after["bytes_" + key] - before["bytes_" + key] == exp[key], key
        _compare_valid([rx, rc, rm, rs, rn], [mx, mc, mm, ms, mn], P)


def test_kmeans_exact_mode_extents(dry):
    """Exact mode (shift = KMEANS_EXACT) takes a sums region of k*d*9 int64 windows (and rejects the
    fixed-point extent k*d), accepts d up to 64, and counts the windows in the reduction bytes."""
    n, d, k = 500, 40, 9
    dry(2)
    hx, hc, hm = np.zeros((n, d), np.float32), np.zeros((k, d), np.float32), np.zeros(n, np.int32)
    hn = np.zeros(k, np.int64)
    rx, rc, rm, rn = (A.accmg_region_create(a) for a in (hx, hc, hm, hn))
    r_small = A.accmg_region_create(np.zeros((k, d), np.int64))
    r_win = A.accmg_region_create(np.zeros((k, d, A.KMEANS_WINDOWS), np.int64))

    def launch(rs, shift):
        A.accmg_loop_launch(A.bounds([0], [n]), A.BODY_KMEANS_ASSIGN,
                            [A.access(rx, A.R, True, d, 0, 0), A.access(rc, A.R), A.access(rm, A.W, True, 1, 0, 0),
                             A.access(rs, A.REDUCE_SUM), A.access(rn, A.REDUCE_SUM)], A.accmg_args_kmeans(n, d, k, shift))
    with pytest.raises(A.AccmgError) as ei:
        launch(r_small, A.KMEANS_EXACT)
    assert ei.value.code == A.EINVAL
    with pytest.raises(A.AccmgError) as ei:
        launch(r_win, 8)  # d = 40 > 32 in fixed-point mode
    assert ei.value.code == A.EUNSUPPORTED
    before = A.accmg_get_stats()["bytes_reduce"]
    launch(r_win, A.KMEANS_EXACT)
    assert A.accmg_get_stats()["bytes_reduce"] - before == 2 * (k * d * A.KMEANS_WINDOWS * 8 + k * 8)
