#!/bin/bash
# Round-2 evidence run (one B200): GPU suite, bench lines, all configs, ncu captures, k-means timeline.
O=${1:-gpurun_out/r02}
mkdir -p $O
python -m pytest tests -m gpu -q -rs > $O/pytest_gpu.log 2>&1
python bench.py > $O/bench.jsonl 2> $O/bench.err
python bench.py --gpus 2 --steps 100 --no-cpu-baseline > $O/bench_gpus2_one_device.jsonl 2> $O/bench2.err
python bench.py --undeclared --steps 50 --no-e2e --no-cpu-baseline > $O/bench_c5.jsonl 2> $O/bench_c5.err
python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.jsonl 2> $O/bench_ref.err
python bench_configs.py --configs c1,c2,c5,c3,c4 --partitions 1,2,4,8 --check > $O/configs.jsonl 2> $O/configs.err
python bench_configs.py --configs f1,f2,f2deep,f3,f4 --partitions 1,2,4,8 > $O/f_rows.jsonl 2> $O/f_rows.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:jacobi2d_tma_k -s 3 -c 1 -o $O/jacobi2d_tma \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:assign_tc -s 1 -c 1 -o $O/kmeans_assign_tc ./scripts/km_prof > /dev/null 2>&1
ncu --set full --clock-control none -k regex:gemm_kernel -s 0 -c 1 -o $O/gemm \
    python bench_configs.py --configs c3 --partitions 1 --gemm-n 16384 --gemm-reps 1 > /dev/null 2>&1
./scripts/km_prof > $O/km_prof.txt
./scripts/km_trace > $O/kmeans_trace_cta0.txt
python scripts/km_trace_summary.py $O/kmeans_trace_cta0.txt > $O/kmeans_trace_summary.txt
for r in jacobi2d_tma kmeans_assign_tc gemm; do ncu -i $O/$r.ncu-rep --page raw --csv > $O/${r}_raw.csv 2>/dev/null; done
python scripts/km_ncu_summary.py $O/kmeans_assign_tc.ncu-rep > $O/kmeans_assign_tc_summary.txt 2>&1
ls -la $O
tail -3 $O/pytest_gpu.log
