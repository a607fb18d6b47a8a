"""GPU parity of the Jacobi loop (configs C1, C2-shape, C5) through the C ABI vs the oracle.

Bit-exact: final arrays, replicas after the exchange, dirty bitmaps, chunk bits, packed buffers,
byte counts (closed forms of SURVEY §8.3 and the oracle's coherence model)."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import bits_of, need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _oracle_run(A0, S):
    A, B = A0.copy(), A0.copy()
    oracle.jacobi_run(A, B, S, nthreads=0)
    return A, B


def _gpu_run(A0, S, P, declared=True, per_loop=False, **kw):
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    A, B = A0.copy(), A0.copy()
    with runtime(num_partitions=P, **kw) as acc:
        per = WL.jacobi_run(A, B, S, declared=declared, per_loop_stats=per_loop)
        st = acc.accmg_get_stats()
    return A, B, per, st


def test_c1_declared_p2_bitexact_and_2048_bytes():
    N, S = 256, 10
    A0 = gen.jacobi_field(1, N)
    oA, oB = _oracle_run(A0, S)
    A, B, per, st = _gpu_run(A0, S, 2, per_loop=True)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    assert all(p["bytes_declared"] == 2048 for p in per[2:])
    assert all(p["bytes_link"] == p["bytes_declared"] for p in per)  # halo rows move as counted
    assert st["body_launches"] == 2 * S


@pytest.mark.parametrize("P", [1, 2, 3, 4, 5, 7, 8])
@pytest.mark.parametrize("halo", ["auto", "pull"])
def test_partition_invariance_bitexact(P, halo):
    """Any partition count gives the 1-partition result bit for bit, with the body pushing its
    boundary rows into the neighbours' replicas (auto: S loops' worth of halo bytes, the last one
    unused) or with pull-before-read only (S - 1 loops' worth)."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    N, S = 1024, 6
    A0 = gen.jacobi_field(2, N)
    oA, oB = _oracle_run(A0, S)
    mode = Acc.HALO_AUTO if halo == "auto" else Acc.HALO_PULL
    A, B, _, st = _gpu_run(A0, S, P, halo_mode=mode)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    if P > 1:
        loops = S if halo == "auto" else S - 1
        assert st["bytes_declared"] == loops * 2 * (P - 1) * 4 * N


@pytest.mark.parametrize("N", [3, 5, 7, 65, 130, 257])
def test_ragged_sizes_scalar_and_vector_paths(N):
    S = 4
    A0 = gen.jacobi_field(3, N)
    A0[:, 0] = 0.75
    oA, oB = _oracle_run(A0, S)
    for P in (1, 3):
        A, B, _, _ = _gpu_run(A0, S, P)
        assert np.array_equal(A, oA) and np.array_equal(B, oB), (N, P)


def test_nccl_self_exchange_matches():
    """exchange_mode = NCCL_ALL: every halo goes through ncclSend/ncclRecv (to self)."""
    N, S = 256, 6
    A0 = gen.jacobi_field(4, N)
    oA, oB = _oracle_run(A0, S)
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    A, B, _, st = _gpu_run(A0, S, 4, exchange_mode=Acc.XCHG_NCCL_ALL)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)


@pytest.mark.parametrize("P,chunk", [(2, 1 << 20), (3, 4096), (1, 1 << 20)])
def test_undeclared_c5_artefacts_bitexact(P, chunk):
    """C5 at C1 size: dirty bitmaps (L133), chunk bits (L135), canonical packed buffers, every
    replica after propagation, byte counts — all bit-exact vs the oracle's model."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    N = 256
    A0 = gen.jacobi_field(1, N)
    A, B = A0.copy(), A0.copy()
    oB = A0.copy()
    bms = oracle.jacobi_sweep(A0, oB, P=P, track=True)
    with runtime(num_partitions=P, debug_checks=1, dirty_chunk_bytes=chunk) as acc:
        rA, rB = acc.accmg_region_create(A), acc.accmg_region_create(B)
        WL.jacobi_sweep(rA, rB, 0, N, False)
        st = acc.accmg_get_stats()
        ce = chunk // 4
        for g in range(P):
            assert np.array_equal(acc.accmg_debug_dirty_bitmap(rB, g), bms[g])
            assert np.array_equal(acc.accmg_debug_chunk_bits(rB, g, ce), oracle.l2_bits(bms[g], N * N, ce))
            assert np.array_equal(acc.accmg_debug_packed(rB, g), oracle.pack(bms[g], oB))
            assert np.array_equal(acc.accmg_debug_replica(rB, g, np.float32).reshape(N, N), oB)
        exp = sum((P - 1) * (16 + 16 * oracle.packed_runs(oracle.pack(b, oB))[0] + 4 * int(bits_of(b, N * N).sum()))
                  for b in bms)
        assert st["bytes_interpartition"] == exp
        if P == 2:
            assert exp == 262160
        acc.accmg_sync_to_host(rB)
        assert np.array_equal(B, oB)


@pytest.mark.parametrize("P", [2, 3])
def test_undeclared_multi_sweep_bitexact(P):
    N, S = 300, 7
    A0 = gen.jacobi_field(5, N)
    oA, oB = _oracle_run(A0, S)
    A, B, per, st = _gpu_run(A0, S, P, declared=False, per_loop=True, dirty_chunk_bytes=8192)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    assert all(p["bytes_interpartition"] == (P - 1) * (16 * P + 16 * (N - 2) + 4 * (N - 2) ** 2) for p in per)
    # the write pass pushes payload only: no run headers, no size words
    assert all(p["bytes_link"] == (P - 1) * 4 * (N - 2) ** 2 for p in per)


def test_undeclared_nccl_self_exchange():
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    N, S = 200, 4
    A0 = gen.jacobi_field(6, N)
    oA, oB = _oracle_run(A0, S)
    A, B, _, _ = _gpu_run(A0, S, 3, declared=False, exchange_mode=Acc.XCHG_NCCL_ALL)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)


def test_sparse_writes_skip_clean_chunks():
    """T9: only every 100th row is written; chunks without dirty rows are skipped (L135)."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    N, P, period, chunk = 1024, 3, 100, 4096
    src = gen.jacobi_field(7, N)
    out0 = gen.jacobi_field(8, N)
    o_out = out0.copy()
    bms = oracle.sparse_rows(src, o_out, period, P=P, track=True)
    out = out0.copy()
    with runtime(num_partitions=P, debug_checks=1, dirty_chunk_bytes=chunk) as acc:
        rs, ro = acc.accmg_region_create(src.copy()), acc.accmg_region_create(out)
        acc.accmg_loop_launch(acc.bounds([0], [N]), Acc.BODY_TEST_SPARSE_WRITE,
                              [acc.access(rs, Acc.R), acc.access(ro, Acc.W)], Acc.accmg_args_sparse(N, N, period))
        st = acc.accmg_get_stats()
        ce = chunk // 4
        for g in range(P):
            assert np.array_equal(acc.accmg_debug_dirty_bitmap(ro, g), bms[g])
            l2 = acc.accmg_debug_chunk_bits(ro, g, ce)
            assert np.array_equal(l2, oracle.l2_bits(bms[g], N * N, ce))
            assert bits_of(l2, N * N // ce).sum() < N * N // ce // 10   # most chunks clean
            assert np.array_equal(acc.accmg_debug_packed(ro, g), oracle.pack(bms[g], o_out))
            assert np.array_equal(acc.accmg_debug_replica(ro, g, np.float32).reshape(N, N), o_out)
        nrows = len(range(0, N, period))
        assert st["bytes_undeclared_payload"] == (P - 1) * nrows * N * 4
        paper = st["bytes_paper_protocol"]
        assert paper > st["bytes_interpartition"]   # whole chunks + bits vs compacted runs


@pytest.mark.parametrize("P,chunk", [(2, 1 << 20), (3, 4096)])
def test_paper_chunk_protocol_bitexact(P, chunk):
    """§8 row f3: the paper's protocol — whole dirty chunks with their L1 bits, merged by the bits
    (L133-135) — gives the same replicas; it moves (P-1) * chunks * (CH*esize + CH/8) bytes."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    N, S = 300, 5
    A0 = gen.jacobi_field(5, N)
    oA, oB = _oracle_run(A0, S)
    A, B, per, st = _gpu_run(A0, S, P, declared=False, per_loop=True, dirty_chunk_bytes=chunk,
                             dirty_protocol=Acc.DIRTY_CHUNKS)
    assert np.array_equal(A, oA) and np.array_equal(B, oB)
    ce = chunk // 4
    for p in per:
        chunks = 0
        for g in range(P):
            a, b = oracle.partition(1, N - 1, P, g)
            chunks += len({e // ce for r in range(a, b) for e in (r * N + 1, r * N + N - 2)} |
                          {c for r in range(a, b) for c in range((r * N + 1) // ce, (r * N + N - 2) // ce + 1)})
        assert p["bytes_interpartition"] == (P - 1) * chunks * (ce * 4 + ce // 8)
        assert p["bytes_link"] == (P - 1) * 4 * (N - 2) ** 2   # the merge stores the dirty elements only


def test_paper_chunk_protocol_sparse_rows():
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    N, P, period, chunk = 1024, 3, 100, 4096
    src = gen.jacobi_field(7, N)
    out0 = gen.jacobi_field(8, N)
    o_out = out0.copy()
    oracle.sparse_rows(src, o_out, period)
    out = out0.copy()
    with runtime(num_partitions=P, dirty_chunk_bytes=chunk, dirty_protocol=Acc.DIRTY_CHUNKS) as acc:
        rs, ro = acc.accmg_region_create(src.copy()), acc.accmg_region_create(out)
        acc.accmg_loop_launch(acc.bounds([0], [N]), Acc.BODY_TEST_SPARSE_WRITE,
                              [acc.access(rs, Acc.R), acc.access(ro, Acc.W)], Acc.accmg_args_sparse(N, N, period))
        for g in range(P):
            assert np.array_equal(acc.accmg_debug_replica(ro, g, np.float32).reshape(N, N), o_out)
        acc.accmg_sync_to_host(ro)
    assert np.array_equal(out, o_out)


@pytest.mark.parametrize("declared", [True, False])
def test_regions_recreated_on_cached_blocks(declared):
    """Regions destroyed and re-created within one runtime reuse the freed device blocks (the
    runtime's block cache holds them by size); the stale contents of a reused block must never
    leak into a result: three fields in turn, each bit-exact, device bytes back to zero each time."""
    N, S = 300, 6
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    with runtime(num_partitions=3) as A:
        for seed in (7, 8, 9):
            A0 = gen.jacobi_field(seed, N)
            Ah, Bh = A0.copy(), A0.copy()
            WL.jacobi_run(Ah, Bh, S, declared=declared)
            oA, oB = _oracle_run(A0, S)
            assert np.array_equal(Ah, oA) and np.array_equal(Bh, oB), seed
            assert A.accmg_get_stats()["device_bytes_user"] == 0
