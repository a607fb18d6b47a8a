#!/bin/bash
# Same-box A/B of the C4 loop: the in-tree library vs paper_conf_icpp_komodamnm13_b200/libaccmg_b.so
# (another build), interleaved, REPS rounds. Usage: scripts/ab_c4.sh [REPS]
REPS=${1:-2}
for rep in $(seq $REPS); do
  for lib in A B; do
    if [ $lib = B ]; then export ACCMG_LIBRARY=$PWD/paper_conf_icpp_komodamnm13_b200/libaccmg_b.so; else unset ACCMG_LIBRARY; fi
    echo -n "$lib "
    timeout 300 python bench_configs.py --configs c4 --partitions 1 --kmeans-iters 6 2>&1 | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(d['ms_per_iteration'])"
  done
done
