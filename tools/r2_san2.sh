#!/bin/bash
# compute-sanitizer on the kernels added late in round 2: forward-plane + TMA, the fused peer-store slabs
set -x
C="fpt_f32_r4 fpt_f64_r3 ps_ws_f32_r2 ps_ip_f32_r2"
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py $C > gpurun_out/san2_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/san2_$tool.log
  tail -4 gpurun_out/san2_$tool.log
done
