#!/bin/bash
# Build the k-means assignment harnesses from the in-tree kernel source: scripts/km_prof (timing /
# ncu target) and scripts/km_trace (clock64 role timeline, -DKM_TRACE). Extra nvcc flags in $1 go
# to both (A/B of build-time variants: scripts/build_km_tools.sh "-DFLAG" SUFFIX).
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
X=${1:-}; S=${2:-}
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -I$ROOT/paper_conf_icpp_komodamnm13_b200/csrc -I$ROOT/include $X"
/usr/local/cuda/bin/nvcc $F -o $ROOT/scripts/km_prof$S $ROOT/scripts/km_trace.cu -lcuda &
/usr/local/cuda/bin/nvcc $F -DKM_TRACE -o $ROOT/scripts/km_trace$S $ROOT/scripts/km_trace.cu -lcuda &
wait
