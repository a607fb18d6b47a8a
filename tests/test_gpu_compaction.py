"""GPU parity of the dirty-bit path with arbitrary write patterns (§8 rows a6-a8; L133-135).

The masked-write test body writes out[e] = in[e] + 1 wherever a seeded mask is set, so the
tracking epilogue, the compaction (count / scan / write passes) and the scatter see isolated bits,
runs crossing word, tile (65536-element) and chunk boundaries, clean tiles between dirty ones,
fully dirty and fully clean arrays, and ragged tails. Every artefact is compared bit-exactly with
the oracle: per-partition L1 bitmaps, chunk bits, canonical packed buffers, every replica after
propagation and the byte counters."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import bits_of, need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


CASES = [  # (n, density, run): sizes span several compaction tiles and end in a ragged tail
    (1000, 0.5, 1),
    (3 * 65536, 1.0, 1),              # fully dirty, tile-aligned
    ((1 << 21) + 12345, 0.5, 1),      # isolated bits: ~n/4 runs
    ((1 << 21) + 77, 0.9, 40),        # runs crossing words
    ((1 << 21) + 5, 0.3, 70001),      # runs crossing tiles and chunks, clean tiles between
    ((1 << 20) + 3, 0.0, 1),          # nothing written
    ((1 << 20) + 31, 0.002, 1),       # very sparse: most chunks clean
]


@pytest.mark.parametrize("n,density,run", CASES)
@pytest.mark.parametrize("P,chunk", [(2, 1 << 20), (3, 4096)])
def test_masked_write_artefacts_bitexact(n, density, run, P, chunk):
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    src = (gen.u_fill(21, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
    mask = gen.write_mask(22, n, density, run)
    out0 = np.full(n, -1.0, dtype=np.float32)
    exp = out0.copy()
    bms = oracle.masked_write(src, mask, exp, P=P, track=True)
    out = out0.copy()
    with runtime(num_partitions=P, debug_checks=1, dirty_chunk_bytes=chunk) as acc:
        ri, rm, ro = acc.accmg_region_create(src), acc.accmg_region_create(mask), acc.accmg_region_create(out)
        acc.accmg_loop_launch(acc.bounds([0], [n]), Acc.BODY_TEST_MASKED_WRITE,
                              [acc.access(ri, Acc.R), acc.access(rm, Acc.R), acc.access(ro, Acc.W)],
                              Acc.accmg_args_masked(n))
        st = acc.accmg_get_stats()
        ce = chunk // 4
        total = 0
        for g in range(P):
            assert np.array_equal(acc.accmg_debug_dirty_bitmap(ro, g), bms[g]), f"bitmap g={g}"
            assert np.array_equal(acc.accmg_debug_chunk_bits(ro, g, ce), oracle.l2_bits(bms[g], n, ce))
            pk = oracle.pack(bms[g], exp)
            assert np.array_equal(acc.accmg_debug_packed(ro, g), pk), f"packed g={g}"
            assert np.array_equal(acc.accmg_debug_replica(ro, g, np.float32), exp), f"replica g={g}"
            nr = oracle.packed_runs(pk)[0]
            total += (P - 1) * (16 + 16 * nr + 4 * int(bits_of(bms[g], n).sum()))
        assert st["bytes_interpartition"] == total
        acc.accmg_sync_to_host(ro)
    assert np.array_equal(out, exp)


def test_masked_write_repeated_loops_clear_bits():
    """Two loops with different masks: the second loop's bitmaps hold only its own writes (the
    compaction cleared L1 and L2 after the first), and the replicas match the oracle's state."""
    from paper_conf_icpp_komodamnm13_b200 import accmg as Acc
    n, P, chunk = (1 << 20) + 999, 3, 8192
    src = (gen.u_fill(31, 0, n) >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
    m1, m2 = gen.write_mask(32, n, 0.7, 5), gen.write_mask(33, n, 0.1, 300)
    exp = np.zeros(n, dtype=np.float32)
    oracle.masked_write(src, m1, exp, P=P)
    bms2 = oracle.masked_write(src, m2, exp, P=P, track=True)
    out = np.zeros(n, dtype=np.float32)
    with runtime(num_partitions=P, debug_checks=1, dirty_chunk_bytes=chunk) as acc:
        ri, ro = acc.accmg_region_create(src), acc.accmg_region_create(out)
        for m in (m1, m2):
            rm = acc.accmg_region_create(m)
            acc.accmg_loop_launch(acc.bounds([0], [n]), Acc.BODY_TEST_MASKED_WRITE,
                                  [acc.access(ri, Acc.R), acc.access(rm, Acc.R), acc.access(ro, Acc.W)],
                                  Acc.accmg_args_masked(n))
            acc.accmg_region_destroy(rm)
        for g in range(P):
            assert np.array_equal(acc.accmg_debug_dirty_bitmap(ro, g), bms2[g])
            assert np.array_equal(acc.accmg_debug_packed(ro, g), oracle.pack(bms2[g], exp))
            assert np.array_equal(acc.accmg_debug_replica(ro, g, np.float32), exp)
