#!/bin/bash
set -x
for c in ps_ws_f32_r2 ps_ip_f32_r2 fpt_f64_r3 ws_f32_r4; do
  timeout 900 compute-sanitizer --tool synccheck --print-limit 5 python tools/sanitize_case.py $c > gpurun_out/san3_$c.log 2>&1
  echo "rc=$?" >> gpurun_out/san3_$c.log
  tail -3 gpurun_out/san3_$c.log
done
