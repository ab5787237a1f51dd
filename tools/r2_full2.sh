#!/bin/bash
set -x
timeout 2700 python -m pytest tests -q -m gpu --timeout 600 > gpurun_out/gputest_full2.log 2>&1; tail -8 gpurun_out/gputest_full2.log
for tool in memcheck racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool python tools/sanitize_case.py ws_f32_r4 ws_f32_r4_full ws_f64_r2 ip_f32_r4 > gpurun_out/san_$tool.log 2>&1
  tail -4 gpurun_out/san_$tool.log
done
