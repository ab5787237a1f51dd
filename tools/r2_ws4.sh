#!/bin/bash
set -x
timeout 60 python tools/ws_smoke.py > gpurun_out/ws4_smoke.log 2>&1; cat gpurun_out/ws4_smoke.log
grep -q "bit-identical to inplane: True" gpurun_out/ws4_smoke.log || exit 1
timeout 300 python tools/tune_one.py --kernel inplane_ws --dtype f32 --top 12 > gpurun_out/ws4_tune.log 2>&1
head -14 gpurun_out/ws4_tune.log
timeout 400 python tools/ab_configs.py --rounds 6 \
  inplane:16,16,4,4,4,2,2,0 inplane:32,8,4,4,4,2,2,0 \
  inplane_ws:32,7,4,2,3,1,4,0 inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,6,2,1,0 \
  > gpurun_out/ws4_ab.json 2> gpurun_out/ws4_ab.err
cat gpurun_out/ws4_ab.json
