"""Pins for the reading behind the tensor-core k-means filter (kmeans_tc.cu header):
the filter computes v ~ V = x.c - |c|^2/2 from bf16 pieces (x = x0 + x1, c = c0 + c1, -|c|^2/2 =
h0 + h1 + h2; products x0.c0 + x0.c1 + x1.c0) accumulated in fp32, claims |v - V| <= E =
2^-11 (L1 Cinf + C2), and re-checks every centroid with v >= vmax - T, T = 2E + 2^-16 Dhat.

Checked here on the CPU, independently of the CUDA code (nothing of it is imported):
  * the emulated filter error (both round-to-nearest and round-toward-zero fp32 accumulation, in
    the MMA's k order and in random orders) stays at least 4x below E on every input family;
  * the exact argmin of the paper's scalar loop (the oracle) is always among the candidates.
CPU only."""
import math

import numpy as np
import pytest

import gen
import oracle


def bf16(a):
    """Round-to-nearest-even fp32 -> bf16, returned as fp32."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32)


def pieces(a):
    h = bf16(a)
    lo = bf16((a - h).astype(np.float32))
    return h, lo


def fp32_accumulate(terms, mode, rng=None):
    """Sequential fp32 accumulation of terms[..., k] (exact fp32 products) in k order or a random
    order; mode 'rn' = round to nearest, 'rz' = round toward zero after every addition."""
    k = terms.shape[-1]
    order = np.arange(k) if rng is None else rng.permutation(k)
    s = np.zeros(terms.shape[:-1], dtype=np.float32)
    for i in order:
        t = s.astype(np.float64) + terms[..., i].astype(np.float64)
        r = t.astype(np.float32)
        if mode == "rz":
            over = np.abs(r.astype(np.float64)) > np.abs(t)
            r = np.where(over, np.nextafter(r, np.float32(0)), r)
        s = r
    return s


def filter_values(x, cen, mode, rng=None):
    """Emulated tensor-core v[p][c] (fp32) for points x [n][16] and centroids cen [k][16]."""
    x0, x1 = pieces(x)
    c0, c1 = pieces(cen)
    q = np.zeros(cen.shape[0], dtype=np.float32)
    for j in range(16):
        q = (q + cen[:, j] * cen[:, j]).astype(np.float32)
    nh = (np.float32(-0.5) * q).astype(np.float32)
    a0 = bf16(nh)
    a1 = bf16((nh - a0).astype(np.float32))
    a2 = bf16((nh - a0 - a1).astype(np.float32))
    # products are exact in fp32 (8-bit x 8-bit significands); K order of the MMA: [x0.c0 | x0.c1 | x1.c0 | h]
    t = np.concatenate([x0[:, None, :] * c0[None, :, :], x0[:, None, :] * c1[None, :, :],
                        x1[:, None, :] * c0[None, :, :],
                        np.broadcast_to(np.stack([a0, a1, a2], -1)[None], (x.shape[0], cen.shape[0], 3))], axis=-1)
    return fp32_accumulate(t.astype(np.float32), mode, rng)


def exact_V(x, cen):
    xd, cd = x.astype(np.float64), cen.astype(np.float64)
    return np.array([[math.fsum(list(xd[p] * cd[c]) + list(-0.5 * cd[c] * cd[c])) for c in range(cen.shape[0])]
                     for p in range(x.shape[0])])


def bound_E(x, cen):
    L1 = np.abs(x.astype(np.float64)).sum(1)
    Cinf = float(np.abs(cen).max())
    C2 = float((cen.astype(np.float64) ** 2).sum(1).max())
    return 2.0 ** -11 * (L1 * Cinf + C2)


def families():
    rng = np.random.default_rng(21)
    lat = gen.kmeans_points(4, 400, 16, 64, gen.KM_LATTICE)
    ovl = gen.kmeans_points(5, 400, 16, 64, gen.KM_OVERLAP)
    small = rng.integers(-2, 3, (400, 16)).astype(np.float32)
    wide = np.round(rng.uniform(-1, 1, (400, 16)) * 2.0 ** rng.integers(0, 21, (400, 1))).astype(np.float32)
    big = (rng.integers(-(2 ** 23) + 1, 2 ** 23, (400, 16)) * 1.0).astype(np.float32)
    mid = (rng.integers(-4, 5, (400, 16)) * 16.0 + 1000.0).astype(np.float32)
    mid[:, 0] = 1001.0 + rng.integers(-3, 4, 400) * np.float32(2.0 ** -8)
    out = []
    for name, pts in (("lattice", lat), ("overlap", ovl), ("small_int", small), ("wide", wide), ("big", big),
                      ("midpoints", mid)):
        # centroids: data points (first iteration) and exact-ish means (later iterations)
        cen_a = pts[:48].copy()
        cen_b = np.stack([pts[i::48].astype(np.float64).mean(0) for i in range(48)]).astype(np.float32)
        out += [(name + "/points", pts, cen_a), (name + "/means", pts, cen_b)]
    return out


@pytest.mark.parametrize("mode", ["rn", "rz"])
@pytest.mark.parametrize("fam", families(), ids=lambda f: f[0])
def test_filter_error_within_E_with_slack(fam, mode):
    _, x, cen = fam
    x = x[:120]
    V = exact_V(x, cen)
    E = bound_E(x, cen)
    for rng in (None, np.random.default_rng(3)):
        v = filter_values(x, cen, mode, rng).astype(np.float64)
        ratio = (np.abs(v - V) / E[:, None]).max()
        assert ratio <= 0.25, f"filter error reaches {ratio:.3f} E"


@pytest.mark.parametrize("fam", families(), ids=lambda f: f[0])
def test_oracle_argmin_is_a_candidate(fam):
    _, x, cen = fam
    v = filter_values(x, cen, "rz").astype(np.float32)
    E = (bound_E(x, cen) * 1.001 + 2.0 ** -100).astype(np.float32)
    Q = (x.astype(np.float32) ** 2).sum(1, dtype=np.float32)
    vmax = v.max(1)
    Dhat = np.maximum(Q * np.float32(1 + 2.0 ** -17) - 2 * vmax + 2 * E, 0).astype(np.float32)
    T = ((2 * E + np.float32(2.0 ** -16) * Dhat) * np.float32(1.001)).astype(np.float32)
    cand = v >= (vmax - T)[:, None]
    truth = oracle.kmeans_assign(np.ascontiguousarray(x), np.ascontiguousarray(cen))
    assert cand[np.arange(x.shape[0]), truth].all()
    # and the candidate sets are small where clusters are separated
    if fam[0].startswith("lattice"):
        assert cand.sum(1).mean() < 2.0
