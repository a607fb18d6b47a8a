"""Stress the multi-process undeclared Jacobi run (tests/mp_worker.py jacobi_undecl, three ranks on
the one GPU) and, on a mismatch, report where the ranks' results differ from the oracle and
whether the wrong values belong to another sweep (stale) or to nothing (garbage)."""
import os
import subprocess
import sys
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
import oracle  # noqa: E402

N, S = 300, 6
A0 = gen.jacobi_field(5, N)
sweeps = [A0.copy()]
a, b = A0.copy(), A0.copy()
for s in range(S):
    src, dst = (a, b) if s % 2 == 0 else (b, a)
    oracle.jacobi_sweep(src, dst)
    sweeps.append(dst.copy())
oA, oB = a, b
world = int(sys.argv[2]) if len(sys.argv) > 2 else 3
work = sys.argv[3] if len(sys.argv) > 3 else "jacobi_undecl"
fails = 0
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 20):
    with tempfile.TemporaryDirectory() as d:
        uid = os.urandom(128).hex()
        ps = [subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "mp_worker.py"), str(r), str(world), "1", uid,
                                work, d, "0", "0", "0"], cwd=ROOT) for r in range(world)]
        rc = [p.wait(timeout=300) for p in ps]
        bad = []
        for r in range(world):
            for name, ref in (("A", oA), ("B", oB)):
                got = np.load(os.path.join(d, f"rank{r}_{name}.npy"))
                diff = np.argwhere(got != ref)
                if len(diff):
                    rows = np.unique(diff[:, 0])
                    src = []
                    for (i, j) in diff[:5]:
                        src.append([k for k, sw in enumerate(sweeps) if sw[i, j] == got[i, j]])
                    bad.append(f"rank {r} {name}: {len(diff)} elements, rows {rows[:10].tolist()}..{rows[-3:].tolist()} "
                               f"(n={len(rows)}), first {diff[:3].tolist()}, matching sweeps {src}")
        print(f"iter {it}: rc {rc} {'OK' if not bad else 'MISMATCH'}", flush=True)
        for l in bad:
            print("   ", l, flush=True)
        fails += bool(bad)
print("fails", fails)
