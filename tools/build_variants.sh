#!/bin/bash
# Build libmars variants that differ only in spmm.cu compile-time parameters
# (dev tool for tools/spmm_ab.py).  Usage: tools/build_variants.sh name "-DFOO=1 ..." ...
set -e
cd "$(dirname "$0")/.."
make -s
mkdir -p build/variants
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -I include -DMARS_BUILD"
others=$(ls build/obj/*.o | grep -v spmm.o)
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  $NV $flags -c paper_conf_icpp_lancl21_b200/csrc/spmm.cu -o build/variants/spmm_$name.o &
done
wait
for o in build/variants/spmm_*.o; do
  n=$(basename $o .o); n=${n#spmm_}
  $NV -shared -o build/variants/libmars_$n.so $others $o -ldl -lpthread -lrt
done
ls build/variants/*.so
