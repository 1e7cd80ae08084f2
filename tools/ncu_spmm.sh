#!/bin/bash
# ncu capture of the SpMM kernels of one bench-config step (bf16 and fp32)
LIB=paper_conf_icpp_lancl21_b200/libmars.so
for p in bf16 fp32; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm -c 5 -o gpurun_out/spmm_$p \
  python tools/step_once.py $LIB $p 1 > gpurun_out/ncu_spmm_$p.log 2>&1; echo "ncu $p rc $?"
done
