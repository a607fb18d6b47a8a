./scripts/km_trace > gpurun_out/kt_a.txt
python -m pytest tests/test_gpu_kmeans_tc.py tests/test_gpu_kmeans.py -q -x 2>&1 | tail -2
./scripts/km_prof | tail -1
python bench_configs.py --configs c4 --partitions 1 --kmeans-iters 6 --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('c4', round(d['ms_per_iteration'],3), d.get('parity'))
    else: print(l.rstrip())"
