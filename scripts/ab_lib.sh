#!/bin/bash
# Same-box A/B of one bench_configs.py config between the in-tree library (A) and
# paper_conf_icpp_komodamnm13_b200/libaccmg_b.so (B), interleaved.
# Usage: scripts/ab_lib.sh "<bench_configs args>" FIELD [REPS]
ARGS="$1"; FIELD="$2"; REPS=${3:-2}
for rep in $(seq $REPS); do
  for side in A B; do
    if [ $side = B ]; then export ACCMG_LIBRARY=$PWD/paper_conf_icpp_komodamnm13_b200/libaccmg_b.so; else unset ACCMG_LIBRARY; fi
    echo -n "$side "
    timeout 300 python bench_configs.py $ARGS 2>&1 | python -c "import sys,json; print([round(json.loads(l)['$FIELD'],4) for l in sys.stdin if l.startswith('{')])"
  done
done
