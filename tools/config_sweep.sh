#!/bin/bash
# Every BASELINE.json config as a bench line on one B200 (run under gpurun):
# gnmt (the metric's workload), inception at b = 1, 4, 16, 64, bert b = 8, and
# the 1.1M-op stress graph unsharded.  Usage: tools/config_sweep.sh TAG
tag=${1:-sweep}
out=gpurun_out/configs_$tag
mkdir -p $out
run() {  # name, args...
  local n=$1; shift
  timeout 900 python bench.py --steps 30 --warmup 5 --no-cpu-baseline "$@" > $out/$n.json 2> $out/$n.err
  echo "$n rc $?"
}
run gnmt --workload gnmt
for b in 1 4 16 64; do run inception_b$b --workload inception --graphs-per-gpu $b; done
run bert_b8 --workload bert
run 1m --workload 1m --steps 10 --no-e2e
