#!/bin/bash
# Same-box A/B of the C3 GEMM: in-tree library vs libaccmg_<name>.so variants, interleaved, REPS
# rounds. Usage: scripts/ab_gemm.sh REPS name...
REPS=$1; shift
for rep in $(seq $REPS); do
  for lib in A "$@"; do
    if [ $lib = A ]; then unset ACCMG_LIBRARY; else export ACCMG_LIBRARY=$PWD/paper_conf_icpp_komodamnm13_b200/libaccmg_$lib.so; fi
    echo -n "$lib "
    timeout 300 python bench_configs.py --configs c3 --partitions 1 --gemm-reps 5 2>&1 | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(round(d['tflops'],1), round(d['ms_per_loop'],3))"
  done
done
