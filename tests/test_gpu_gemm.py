"""GPU parity of the matmul loop (config C3 shape) through the C ABI vs the fp64 oracle.

Integer-valued bf16 inputs in {-2..2}: every partial sum is an integer below 2^24, so the fp32
tensor-core result equals (float) of the exact fp64 oracle bit for bit, in any accumulation order
(reading W3(i)). Uniform (0,1] inputs: elementwise relative error <= 1e-2 (north star)."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import need_gpu, runtime

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _gpu():
    need_gpu()


def _run(Ab, Bb, P, **kw):
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    from paper_conf_icpp_komodamnm13_b200 import workloads as WL
    M, K = Ab.shape
    N = Bb.shape[1]
    C = np.zeros((M, N), dtype=np.float32)
    with runtime(num_partitions=P, **kw) as acc:
        ra, rb, rc = acc.accmg_region_create(Ab), acc.accmg_region_create(Bb), acc.accmg_region_create(C)
        WL.gemm_loop(ra, rb, rc, M, N, K)
        acc.accmg_sync_to_host(rc)
        st = acc.accmg_get_stats()
    return C, st


@pytest.mark.parametrize("M,N,K,P", [(128, 256, 64, 1), (256, 512, 256, 1), (300, 256, 128, 3), (1000, 768, 640, 4),
                                     (129, 256, 64, 2)])
def test_integer_inputs_bitexact(M, N, K, P):
    Ab = gen.bf16_matrix(3, M, K, gen.BF16_INTS)
    Bb = gen.bf16_matrix(4, K, N, gen.BF16_INTS)
    C, st = _run(Ab, Bb, P)
    R = oracle.gemm_rows_f64(Ab, Bb, np.arange(M))
    assert np.array_equal(C, R.astype(np.float32))
    assert st["bytes_declared"] == 0          # A rows and C rows are pulled from the host only


def test_identity_and_partition_invariance():
    M, K = 512, 512
    Ab = gen.bf16_matrix(5, M, K, gen.BF16_UNIT)
    I = (np.eye(K, dtype=np.float32).view(np.uint32) >> 16).astype(np.uint16)
    C, _ = _run(Ab, I, 3)
    assert np.array_equal(C, gen.bf16_to_f32(Ab))
    Bb = gen.bf16_matrix(6, K, 256, gen.BF16_UNIT)
    C1, _ = _run(Ab, Bb, 1)
    C5, _ = _run(Ab, Bb, 5)
    assert np.array_equal(C1, C5)            # fixed k order per element (W9)


def test_uniform_inputs_tolerance():
    M, N, K = 1024, 1024, 2048
    Ab = gen.bf16_matrix(7, M, K, gen.BF16_UNIT)
    Bb = gen.bf16_matrix(8, K, N, gen.BF16_UNIT)
    C, _ = _run(Ab, Bb, 2)
    rows = np.array([0, 1, 127, 128, 511, 512, 1000, 1023])
    R = oracle.gemm_rows_f64(Ab, Bb, rows)
    rel = np.abs(C[rows] - R) / np.abs(R)
    assert rel.max() <= 1e-2
    assert rel.max() <= 1e-5                 # fp32 accumulation of positive terms: ~1e-6 expected


def test_large_sampled_rows():
    M, N, K = 4096, 4096, 4096
    Ab = gen.bf16_matrix(9, M, K, gen.BF16_INTS)
    Bb = gen.bf16_matrix(10, K, N, gen.BF16_INTS)
    C, _ = _run(Ab, Bb, 4)
    rows = np.unique(np.concatenate([np.arange(0, M, 97), [M - 1, 1023, 1024, 2047, 2048, 3071, 3072]]))
    R = oracle.gemm_rows_f64(Ab, Bb, rows)
    assert np.array_equal(C[rows], R.astype(np.float32))


@pytest.mark.parametrize("N,P", [(8, 1), (136, 3), (272, 1), (272, 2), (1000, 3)])
def test_partial_last_n_block_bitexact(N, P):
    """N not a multiple of the 256-column tile: the last n-block's B columns past N are zero-filled
    by the TMA and its accumulators past N are not stored (N % 8 == 0)."""
    M, K = 300, 128
    Ab = gen.bf16_matrix(11, M, K, gen.BF16_INTS)
    Bb = gen.bf16_matrix(12, K, N, gen.BF16_INTS)
    C, _ = _run(Ab, Bb, P)
    R = oracle.gemm_rows_f64(Ab, Bb, np.arange(M))
    assert np.array_equal(C, R.astype(np.float32))


@pytest.mark.parametrize("N,K", [(12, 64), (256, 96)])
def test_unsupported_shapes_rejected(N, K):
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    M = 128
    Ab = gen.bf16_matrix(13, M, K, gen.BF16_INTS)
    Bb = gen.bf16_matrix(14, K, N, gen.BF16_INTS)
    with pytest.raises(A.AccmgError) as ei:
        _run(Ab, Bb, 1)
    assert ei.value.code == A.EUNSUPPORTED


def test_uniform_inputs_full_4096():
    """T11 in full: every element of a 4096^3 uniform (0,1] bf16 product against the fp64 oracle,
    elementwise relative error <= 1e-2 (north star; fp32 accumulation of positive terms gives ~1e-6)."""
    M = N = K = 4096
    Ab = gen.bf16_matrix(15, M, K, gen.BF16_UNIT)
    Bb = gen.bf16_matrix(16, K, N, gen.BF16_UNIT)
    C, _ = _run(Ab, Bb, 2)
    R = oracle.gemm_rows_f64(Ab, Bb, np.arange(M))
    rel = np.abs(C - R) / np.abs(R)
    assert rel.max() <= 1e-2
    # positive terms: fp32 accumulation in any order (and rounding mode) is within (K - 1) 2^-23
    assert rel.max() <= (K - 1) * 2.0 ** -23


def test_uniform_inputs_sampled_32768():
    """T11 at the C3 size: 32768^3 uniform (0,1] bf16, 64 sampled rows (the first and last row of
    every partition at P = 4 plus spread rows) against the fp64 oracle."""
    M = N = K = 32768
    Ab = gen.bf16_matrix(17, M, K, gen.BF16_UNIT)
    Bb = gen.bf16_matrix(18, K, N, gen.BF16_UNIT)
    C, _ = _run(Ab, Bb, 4)
    edges = [0, 8191, 8192, 16383, 16384, 24575, 24576, 32767]
    rows = np.unique(np.concatenate([edges, np.linspace(1, M - 2, 56).astype(np.int64)]))
    R = oracle.gemm_rows_f64(Ab, Bb, rows)
    rel = np.abs(C[rows] - R) / np.abs(R)
    assert rel.max() <= 1e-2
    assert rel.max() <= (K - 1) * 2.0 ** -23
