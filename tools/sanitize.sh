#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over
# tools/sanitize_steps.py (run under gpurun); logs into gpurun_out/sanitize_<tool>.txt
# TOOLS="memcheck initcheck" MARS_SAN_ONLY=variants tools/sanitize.sh  runs a subset
for t in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 50 --error-exitcode 9 \
    python tools/sanitize_steps.py > gpurun_out/sanitize_$t.txt 2>&1
  echo "$t rc $?"
  tail -3 gpurun_out/sanitize_$t.txt
done
