"""ORACLE — TEST INFRASTRUCTURE ONLY: brute-force per-element coherence model.

Tracks, for every element of every region, on which partitions (and on the host) the
current value is held, and counts the bytes each step must move. It is the "obviously
correct" reference for the product's interval-based validity table, pull planner and byte
counters. Per-element boolean arrays: for small extents only.

Semantics followed (PAPER.md line numbers; readings from SURVEY §8.3 / DESIGN.md):
  * placement: arrays with a localaccess window are distributed — a partition needs only the
    union of its iterations' windows (L121-123, L87); arrays without one are replicated on every
    partition (L121, "the default placement policy");
  * data loader: before every loop, load what each partition may read and is not already valid
    there (L119, L125 reload elision); the writer's replica must be valid on its whole declared
    write window (G16);
  * declared writes: the writer becomes the only valid holder of its write window (owner
    computes; windows of different partitions are disjoint, G14);
  * undeclared writes: every partition's dirty elements are propagated to all other replicas
    right after the loop (L129-133), costing (P-1) * (16 + 16*runs + esize*elems) bytes per
    sender (canonical packed buffer);
  * reductiontoarray destinations: replicated; partial results merged across partitions
    (L112), counted as a ring all-reduce: 2(P-1) * extent * esize bytes (reading W8).
"""
from __future__ import annotations

import numpy as np

from . import partition, window_iter

R, W, RW, REDUCE_SUM = 1, 2, 3, 4


class Region:
    def __init__(self, extent: int, esize: int, P: int):
        self.extent, self.esize = extent, esize
        self.valid = np.zeros((P, extent), dtype=bool)
        self.host_valid = np.ones(extent, dtype=bool)


def _runs(mask: np.ndarray) -> int:
    m = mask.astype(np.int8)
    return int(np.count_nonzero(np.diff(np.concatenate(([0], m))) == 1))


class Model:
    def __init__(self, P: int, chunk_bytes: int = 1 << 20):
        self.P, self.chunk_bytes = P, chunk_bytes
        self.stats = dict(interpartition=0, declared=0, undeclared_payload=0, undeclared_headers=0,
                          reduce=0, h2d=0, d2h=0, paper_protocol=0, loops=0)

    def region(self, extent: int, esize: int) -> Region:
        return Region(extent, esize, self.P)

    def window(self, a: int, b: int, stride: int, left: int, right: int, extent: int) -> np.ndarray:
        """Union over iterations i in [a, b) of the per-iteration window (L87), clipped."""
        m = np.zeros(extent, dtype=bool)
        for i in range(a, b):
            lo, hi = window_iter(stride, left, right, i)
            m[max(lo, 0):max(min(hi, extent), 0)] = True
        return m

    def loop(self, lo: int, hi: int, descs, written=None) -> dict:
        """descs: (region, mode, declared, stride, left, right); written: {id(region): [P masks]}
        for undeclared written regions. Returns this loop's byte counts."""
        P = self.P
        chunks = [partition(lo, hi, P, g) for g in range(P)]
        out = dict(interpartition=0, declared=0, undeclared_payload=0, undeclared_headers=0,
                   reduce=0, h2d=0, paper_protocol=0)
        needs = []
        for (rg, mode, decl, s, l, r) in descs:
            if decl and mode != REDUCE_SUM:
                need = [self.window(a, b, s, l, r, rg.extent) for (a, b) in chunks]
            else:
                need = [np.ones(rg.extent, dtype=bool) for _ in range(P)]
            needs.append(need)
        # data loader: pull-before-read
        # sources are chosen from the state before the pull phase (all pulls of a phase are
        # planned together and run concurrently)
        for (rg, mode, decl, s, l, r), need in zip(descs, needs):
            held = rg.valid.any(axis=0)
            for g in range(P):
                miss = need[g] & ~rg.valid[g]
                on_peer = miss & held
                from_host = miss & ~on_peer
                assert np.all(rg.host_valid[from_host]), "element valid nowhere"
                nb = int(np.count_nonzero(on_peer)) * rg.esize
                out["interpartition"] += nb
                out["declared"] += nb
                out["h2d"] += int(np.count_nonzero(from_host)) * rg.esize
                rg.valid[g] |= need[g]
        # after the loop: coherence
        for (rg, mode, decl, s, l, r), need in zip(descs, needs):
            if mode == REDUCE_SUM:
                nb = 2 * (P - 1) * rg.extent * rg.esize
                out["reduce"] += nb
                out["interpartition"] += nb
                rg.host_valid[:] = False
                continue
            if not (mode & W):
                continue
            if decl:
                for g in range(P):
                    wg = need[g]
                    for h in range(g):
                        assert not np.any(wg & need[h]), "overlapping declared write windows (G14)"
                for g in range(P):
                    wg = need[g]
                    rg.valid[:, wg] = False
                    rg.valid[g, wg] = True
                    rg.host_valid[wg] = False
            else:
                masks = written[id(rg)]
                ch = self.chunk_bytes // rg.esize
                for g in range(P):
                    wm = masks[g]
                    runs, elems = _runs(wm), int(np.count_nonzero(wm))
                    out["undeclared_headers"] += (P - 1) * (16 + 16 * runs)
                    out["undeclared_payload"] += (P - 1) * elems * rg.esize
                    out["interpartition"] += (P - 1) * (16 + 16 * runs + elems * rg.esize)
                    nchunks = len(np.unique(np.nonzero(wm)[0] // ch)) if elems else 0
                    out["paper_protocol"] += (P - 1) * nchunks * (ch * rg.esize + ch // 8)
                # the host copy is treated as stale as a whole: the dirty sets live on the devices
                rg.host_valid[:] = False
        for k, v in out.items():
            self.stats[k] += v
        self.stats["loops"] += 1
        return out

    def sync_to_host(self, rg: Region) -> int:
        nb = int(np.count_nonzero(~rg.host_valid)) * rg.esize
        rg.host_valid[:] = True
        self.stats["d2h"] += nb
        return nb
