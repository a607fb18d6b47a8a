#!/bin/bash
# Build paper_conf_icpp_komodamnm13_b200/libaccmg_<NAME>.so: the in-tree objects with one source
# recompiled under extra flags (same-box A/B of kernel variants through ACCMG_LIBRARY).
# Usage: scripts/build_variant.sh NAME SOURCE.cu "-DFLAG ..."   (run `make accmg` first)
set -e
NAME=$1; SRC=$2; FLAGS=$3
ROOT=$(cd "$(dirname "$0")/.." && pwd)
PKG=$ROOT/paper_conf_icpp_komodamnm13_b200
NCCL_INC=$(python -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null || true)
mkdir -p $ROOT/build/var/$NAME
base=$(basename $SRC .cu)
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 \
  --expt-relaxed-constexpr -I$ROOT/include -I$PKG/csrc ${NCCL_INC:+-I$NCCL_INC} $FLAGS -c -o $ROOT/build/var/$NAME/$base.o $PKG/csrc/$base.cu
objs=$(ls $ROOT/build/obj/*.o | grep -v "/$base.o$")
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $PKG/libaccmg_$NAME.so $ROOT/build/var/$NAME/$base.o $objs -lcudart_static -ldl -lrt -lpthread
echo built $PKG/libaccmg_$NAME.so
