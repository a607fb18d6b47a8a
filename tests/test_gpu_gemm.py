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


@pytest.mark.skipif(bool(__import__("os").environ.get("ACCMG_GEMM_IMPL")), reason="already a per-impl run")
def test_two_sm_variant_bitexact():
    """ACCMG_GEMM_IMPL=2 (tcgen05.mma.cta_group::2 CTA pairs), read once per process: the GEMM
    tests in a child process."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider", "tests/test_gpu_gemm.py",
                        "-k", "not two_sm_variant"], cwd=root, env=dict(os.environ, ACCMG_GEMM_IMPL="2"),
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:]
