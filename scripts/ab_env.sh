#!/bin/bash
# Same-box A/B of the C4 loop between two environment settings, interleaved.
# Usage: scripts/ab_env.sh "ENV_A" "ENV_B" [REPS]    e.g. scripts/ab_env.sh "" "ACCMG_KMEANS_TC_SETS=2" 2
A="$1"; B="$2"; REPS=${3:-2}
for rep in $(seq $REPS); do
  for side in A B; do
    if [ $side = A ]; then E="$A"; else E="$B"; fi
    echo -n "$side [$E] "
    env $E timeout 300 python bench_configs.py --configs c4 --partitions 1 --kmeans-iters 6 2>&1 | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(d['ms_per_iteration'])"
  done
done
