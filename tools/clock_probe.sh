#!/bin/bash
# Dev tool: nvidia-smi clocks / power / throttle reasons sampled every 20 ms
# while tools/step_series.py runs the bench step (is the step-time rise after
# the first ~15 steps a clock change?).  Output: gpurun_out/clock_probe.csv
nvidia-smi --query-gpu=timestamp,clocks.sm,clocks.mem,power.draw,temperature.gpu,temperature.memory,clocks_throttle_reasons.active --format=csv -lms 20 > gpurun_out/clock_probe.csv &
pid=$!
sleep 1
timeout 300 python tools/step_series.py paper_conf_icpp_lancl21_b200/libmars.so
sleep 1
kill $pid
