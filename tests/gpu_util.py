"""Shared helpers of the -m gpu tests: import the product binding only when a GPU test runs."""
import contextlib

import pytest


def need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@contextlib.contextmanager
def runtime(**kw):
    from paper_conf_icpp_komodamnm13_b200 import accmg as A
    kw.setdefault("device", 0)
    A.accmg_init(**kw)
    try:
        yield A
    finally:
        A.accmg_finalize()


def bits_of(words, extent):
    import numpy as np
    return np.unpackbits(np.ascontiguousarray(words).view(np.uint8), bitorder="little")[:extent].astype(bool)
