#!/bin/bash
# Build libmars variants that differ only in spmm.cu compile-time parameters
# (dev tool for tools/spmm_ab.py).  Usage: [SRC=head] tools/build_variants.sh name "-DFOO=1 ..." ...
# SRC selects the translation unit that is recompiled (default spmm).
set -e
cd "$(dirname "$0")/.."
make -s
mkdir -p build/variants
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -I include -DMARS_BUILD"
SRC=${SRC:-spmm}
others=$(ls build/obj/*.o | grep -v "/$SRC.o")
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  $NV $flags -c paper_conf_icpp_lancl21_b200/csrc/$SRC.cu -o build/variants/${SRC}_$name.o &
done
wait
for o in build/variants/${SRC}_*.o; do
  n=$(basename $o .o); n=${n#${SRC}_}
  $NV -shared -o build/variants/libmars_$n.so $others $o -ldl -lpthread -lrt
done
ls build/variants/*.so
