#!/bin/bash
# Dev tool: ncu --set full --import-source capture of ONE launch of each named
# kernel of a bench-config fp32 step, with the per-SASS-line stall samples as
# CSV (gpurun_out/src_<name>.csv).  Usage: tools/ncu_source.sh name:regex:skip ...
LIB=paper_conf_icpp_lancl21_b200/libmars.so
for spec in "$@"; do
  IFS=: read name rx skip <<< "$spec"
  timeout 600 ncu --set full --import-source on --clock-control none -k "regex:$rx" \
    --launch-skip ${skip:-0} -c 1 -f -o /tmp/src_$name python tools/step_once.py $LIB ${PREC:-fp32} 1 \
    > /dev/null 2>&1; echo "$name rc $?"
  ncu -i /tmp/src_$name.ncu-rep --page source --csv --print-source sass > gpurun_out/src_$name.csv 2>&1
done
