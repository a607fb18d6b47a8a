#!/bin/bash
# Same-box A/B of km_prof builds (interleaved, 3 rounds): scripts/r2_kab.sh SUFFIX...
for r in 1 2 3; do
  for s in "$@"; do
    [ "$s" = "-" ] && s=""
    echo "km_prof$s $(timeout 60 ./scripts/km_prof$s | tail -1)"
  done
done
