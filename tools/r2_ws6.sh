#!/bin/bash
set -x
gunzip -k -f tools/variants/ws5.so.gz
timeout 60 python tools/ws_smoke.py > gpurun_out/ws6_smoke.log 2>&1; cat gpurun_out/ws6_smoke.log
grep -q "bit-identical to inplane: True" gpurun_out/ws6_smoke.log || exit 1
timeout 300 python tools/tune_one.py --kernel inplane_ws --dtype f32 --top 12 > gpurun_out/ws6_tune.log 2>&1
head -8 gpurun_out/ws6_tune.log
C="inplane:16,16,4,4,4,2,2,0 inplane:16,15,4,4,4,2,2,0 inplane_ws:16,16,4,2,6,1,2,0 inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:16,16,4,4,6,2,1,0"
for i in 1 2; do
  STENCIL_LIB=tools/variants/ws5.so timeout 200 python tools/ab_configs.py --rounds 4 $C > gpurun_out/ws6_old_$i.json 2>/dev/null
  timeout 200 python tools/ab_configs.py --rounds 4 $C > gpurun_out/ws6_new_$i.json 2>/dev/null
done
