#!/bin/bash
# One gpurun call: k-means parity, timing (C4 at P = 1), timeline and an ncu capture of assign_tc.
# Usage (on the box): scripts/r2_km2.sh TAG
T=${1:-x}
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_kmeans_tc.py tests/test_gpu_kmeans.py -q -x 2>&1 | tail -3
timeout 60 ./scripts/km_prof | tail -1
timeout 300 python bench_configs.py --configs c4 --partitions 1 --kmeans-iters 6 --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('c4', round(d['ms_per_iteration'],3), d.get('parity'), d.get('assign_frac_of_tensor_bound'))
    else: print(l.rstrip())"
timeout 60 ./scripts/km_trace > gpurun_out/kt_$T.txt; python scripts/km_trace_summary.py gpurun_out/kt_$T.txt | head -40
timeout 300 ncu --set full --clock-control none --import-source on -k regex:assign_tc -s 1 -c 1 -o gpurun_out/km_$T ./scripts/km_prof > /dev/null 2>&1
ls -la gpurun_out/km_$T*
