"""Pins for the oracle's task mapping, windows, dirty-bit/packing model and byte model.

Each check is fixed by the paper's prose or by mathematics, never by re-calling the oracle's
own formula: brute force over iterations, naive run search, closed forms and the C1 worked
example of SURVEY §8.3. CPU only.
"""
import numpy as np
import pytest

import oracle
from oracle import model as M


# ---- L108: equal division (reading G6) ------------------------------------------------------
@pytest.mark.parametrize("P", range(1, 10))
def test_partition_cover_contiguous_balanced(P):
    for lo in (0, 1, 5):
        for n in range(0, 65):
            hi = lo + n
            chunks = [oracle.partition(lo, hi, P, g) for g in range(P)]
            assert chunks[0][0] == lo and chunks[-1][1] == hi
            for g in range(P - 1):
                assert chunks[g][1] == chunks[g + 1][0]          # contiguous, ordered by g
            sizes = [b - a for a, b in chunks]
            assert sum(sizes) == n and max(sizes) - min(sizes) <= 1   # "equally divided"
            for i in range(lo, hi):                               # every task exactly once
                owners = [g for g, (a, b) in enumerate(chunks) if a <= i < b]
                assert owners == [oracle.owner(lo, hi, P, i)]


def test_partition_c1_worked_example():
    # N=256 rows [1,255), P=2 -> g0 = [1,128), g1 = [128,255)
    assert oracle.partition(1, 255, 2, 0) == (1, 128)
    assert oracle.partition(1, 255, 2, 1) == (128, 255)


# ---- L87: localaccess window ----------------------------------------------------------------
def test_window_iter_literal_examples():
    # "from stride*i - left to stride*(i+1) - 1 + right" (inclusive) -> half-open [lo, hi+1)
    assert oracle.window_iter(1, 0, 0, 5) == (5, 6)
    assert oracle.window_iter(4, 1, 2, 3) == (11, 18)        # [12-1, 16-1+2] = [11, 17]
    assert oracle.window_iter(256, 256, 256, 1) == (0, 768)  # Jacobi row 1 reads rows 0..2


def test_c1_windows_worked_example():
    mdl = M.Model(2)
    N, E = 256, 256 * 256
    r0 = mdl.window(1, 128, N, N, N, E)
    r1 = mdl.window(128, 255, N, N, N, E)
    assert np.flatnonzero(r0)[[0, -1]].tolist() == [0, 33023]
    assert np.flatnonzero(r1)[[0, -1]].tolist() == [32512, 65535]
    w0 = mdl.window(1, 128, N, 0, 0, E)
    w1 = mdl.window(128, 255, N, 0, 0, E)
    assert np.flatnonzero(w0)[[0, -1]].tolist() == [256, 32767] and w0.sum() == 32768 - 256
    assert np.flatnonzero(w1)[[0, -1]].tolist() == [32768, 65279]


# ---- L133-135: dirty bits, chunk bits, canonical packing -------------------------------------
def _naive_runs(bits):
    runs, e = [], 0
    while e < len(bits):
        if bits[e]:
            s = e
            while e < len(bits) and bits[e]:
                e += 1
            runs.append((s, e))
        else:
            e += 1
    return runs


def _to_words(bits):
    E = len(bits)
    w = np.zeros((E + 31) // 32, dtype=np.uint32)
    for e in np.flatnonzero(bits):
        w[e // 32] |= np.uint32(1 << (e % 32))
    return w


@pytest.mark.parametrize("seed", range(40))
def test_pack_vs_naive_runs(seed):
    rng = np.random.default_rng(seed)
    E = int(rng.integers(1, 400))
    density = rng.choice([0.02, 0.3, 0.7, 0.98])
    bits = rng.random(E) < density
    vals = rng.standard_normal(E).astype(np.float32)
    pk = oracle.pack(_to_words(bits), vals)
    nr, ne, rs, re, pay = oracle.packed_runs(pk)
    runs = _naive_runs(bits)
    assert nr == len(runs) and ne == int(bits.sum())
    assert rs.tolist() == [a for a, _ in runs] and re.tolist() == [b for _, b in runs]
    assert np.array_equal(pay.view(np.float32), vals[bits])
    assert pk.size == 16 + 16 * nr + 4 * ne
    dst = np.zeros(E, dtype=np.float32)
    oracle.unpack(pk, dst)
    assert np.array_equal(dst[bits], vals[bits]) and np.all(dst[~bits] == 0)


def test_l2_bits_brute_force():
    rng = np.random.default_rng(1)
    E, ch = 5000, 256
    bits = np.zeros(E, dtype=bool)
    bits[rng.integers(0, E, 7)] = True
    l2 = oracle.l2_bits(_to_words(bits), E, ch)
    expect = {e // ch for e in np.flatnonzero(bits)}
    got = {c for c in range((E + ch - 1) // ch) if (int(l2[c // 32]) >> (c % 32)) & 1}
    assert got == expect


# ---- byte model: closed forms and the C1 worked example ---------------------------------------
def _jacobi_loop(mdl, regs, s, N, declared, P):
    src, dst = regs[s % 2], regs[(s + 1) % 2]
    if declared:
        descs = [(src, M.R, 1, N, N, N), (dst, M.W, 1, N, 0, 0)]
        written = None
    else:
        descs = [(src, M.R, 0, 0, 0, 0), (dst, M.W, 0, 0, 0, 0)]
        masks = []
        for g in range(P):
            a, b = oracle.partition(1, N - 1, P, g)
            m = np.zeros((N, N), dtype=bool)
            m[a:b, 1:N - 1] = True
            masks.append(m.reshape(-1))
        written = {id(dst): masks}
    return mdl.loop(1, N - 1, descs, written)


def test_c1_declared_2048_bytes_per_sweep():
    N, P = 256, 2
    mdl = M.Model(P)
    regs = [mdl.region(N * N, 4), mdl.region(N * N, 4)]
    per = [_jacobi_loop(mdl, regs, s, N, True, P) for s in range(10)]
    assert all(p["interpartition"] == 2048 for p in per[2:])
    assert per[0]["interpartition"] == 0                 # sweep 0: everything from the host
    assert per[0]["h2d"] > 0 and all(p["h2d"] == 0 for p in per[2:])


def test_c1_undeclared_262160_bytes_per_sweep():
    N, P = 256, 2
    mdl = M.Model(P)
    regs = [mdl.region(N * N, 4), mdl.region(N * N, 4)]
    per = [_jacobi_loop(mdl, regs, s, N, False, P) for s in range(4)]
    assert all(p["interpartition"] == 262160 for p in per)
    assert per[0]["undeclared_headers"] == 2 * (16 + 127 * 16)
    assert 262160 // 2048 == 128


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_byte_closed_forms(P):
    N = 48
    mdl = M.Model(P, chunk_bytes=1024)
    regs = [mdl.region(N * N, 4), mdl.region(N * N, 4)]
    decl = [_jacobi_loop(mdl, regs, s, N, True, P) for s in range(6)][3:]
    assert all(p["interpartition"] == 2 * (P - 1) * 4 * N for p in decl)
    mdl2 = M.Model(P, chunk_bytes=1024)
    regs2 = [mdl2.region(N * N, 4), mdl2.region(N * N, 4)]
    und = [_jacobi_loop(mdl2, regs2, s, N, False, P) for s in range(3)]
    assert all(p["interpartition"] == (P - 1) * (16 * P + 16 * (N - 2) + 4 * (N - 2) ** 2) for p in und)
