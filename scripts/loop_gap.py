"""Per-loop time vs body time: C2 declared at P = 1 and 8 virtual partitions, profile off / on.
Prints one JSON line per case: ms per loop from CUDA events around the loop sequence (library
stream), and ms_body from the library's per-phase events when profile = 1."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import accmg as A  # noqa: E402
from paper_conf_icpp_komodamnm13_b200 import workloads as WL  # noqa: E402

N = int(os.environ.get("GAP_N", "32768"))
loops = int(os.environ.get("GAP_LOOPS", "60"))
for P in (1, 8):
    for prof in (0, 1):
        A.accmg_init(num_partitions=P, device=0, profile=prof)
        Ah = gen.jacobi_field(2, N)
        Bh = Ah.copy()
        rA, rB = A.accmg_region_create(Ah), A.accmg_region_create(Bh)
        for s in range(6):
            WL.jacobi_sweep(rA, rB, s, N, True)
        A.accmg_barrier()
        A.accmg_reset_stats()
        st = torch.cuda.ExternalStream(A.accmg_stream(), device=0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for s in range(6, 6 + loops):
            WL.jacobi_sweep(rA, rB, s, N, True)
        e1.record(st)
        A.accmg_barrier()
        ms = e0.elapsed_time(e1) / loops
        s_ = A.accmg_get_stats()
        print(json.dumps({"P": P, "profile": prof, "ms_per_loop": round(ms, 5),
                          "ms_body": round(s_["ms_body"] / loops, 5) if prof else None,
                          "gap_us": round((ms - s_["ms_body"] / loops) * 1e3, 2) if prof else None,
                          "env": {k: v for k, v in os.environ.items() if k.startswith("ACCMG_")}}), flush=True)
        A.accmg_region_destroy(rA)
        A.accmg_region_destroy(rB)
        A.accmg_finalize()
