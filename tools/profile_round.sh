#!/bin/bash
# Round-end evidence on one B200 (run under gpurun): full bench line, the
# reference (oracle) arm, the ncu launch list of the bench command, and one
# `ncu --set full` capture of every kernel of one fp32 and one bf16 step.
# Usage: tools/profile_round.sh TAG
tag=${1:-r1}
out=gpurun_out/$tag
mkdir -p $out
timeout 600 python bench.py > $out/bench.json 2> $out/bench.err; echo "bench rc $?"
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > $out/reference.json 2> $out/reference.err; echo "ref rc $?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1; echo "launches rc $?"
LIB=paper_conf_icpp_lancl21_b200/libmars.so
K='regex:k_tc3h_rows|k_tc3h_dw|k_tc16_rows|k_tc16_dw|k_spmm_fwd|k_spmm_bwd|k_dz3|k_score|k_colsum'
rep=${NCU_REP_DIR:-/tmp}    # large .ncu-rep files stay on the box; summaries come back
timeout 900 ncu --set full --clock-control none --import-source on -f -k "$K" -c 17 -o $rep/full_fp32 \
  python tools/step_once.py $LIB fp32 1 > /dev/null 2>&1; echo "full fp32 rc $?"
timeout 900 ncu --set full --clock-control none --import-source on -f -k "$K" -c 17 -o $rep/full_bf16 \
  python tools/step_once.py $LIB bf16 1 > /dev/null 2>&1; echo "full bf16 rc $?"
python tools/ncu_table.py $rep/full_fp32.ncu-rep > $out/ncu_full_fp32.txt 2>&1
python tools/ncu_table.py $rep/full_bf16.ncu-rep > $out/ncu_full_bf16.txt 2>&1
python tools/traffic_from_ncu.py $tag $rep/full_fp32.ncu-rep $rep/full_bf16.ncu-rep && cp profiles/${tag}_traffic.json $out/
ls -la $out
