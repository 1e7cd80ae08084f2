#!/bin/bash
# GPU test run: full -m gpu suite, summary into gpurun_out/tests_<tag>.txt
tag=${1:-x}
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -rf -s > gpurun_out/tests_$tag.txt 2>&1
echo "pytest rc $?"
grep -E "^E |FAILED|passed|failed|stage-wise|TIMING" gpurun_out/tests_$tag.txt | head -40
