#!/bin/bash
# Like build_variants.sh, for variants that recompile several translation units:
# SRCS="gemm_tc3h head" tools/build_variants2.sh name "-DFOO=1" ...
set -e
cd "$(dirname "$0")/.."
make -s
mkdir -p build/variants
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -I include -DMARS_BUILD"
SRCS=${SRCS:-spmm}
others=$(ls build/obj/*.o)
for src in $SRCS; do others=$(echo "$others" | grep -v "/$src.o"); done
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  objs=""
  for src in $SRCS; do
    $NV $flags -c paper_conf_icpp_lancl21_b200/csrc/$src.cu -o build/variants/${src}_$name.o &
    objs="$objs build/variants/${src}_$name.o"
  done
  wait
  $NV -shared -o build/variants/libmars_$name.so $others $objs -ldl -lpthread -lrt
done
ls build/variants/*.so
