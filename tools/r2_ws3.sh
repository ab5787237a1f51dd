#!/bin/bash
set -x
timeout 60 python tools/ws_smoke.py > gpurun_out/ws3_smoke.log 2>&1; cat gpurun_out/ws3_smoke.log
grep -q "bit-identical to inplane: True" gpurun_out/ws3_smoke.log || exit 1
timeout 400 python tools/ab_configs.py --rounds 6 \
  inplane:16,16,4,4,4,2,2,0 inplane:32,8,4,4,4,2,2,0 inplane:32,7,4,2,4,1,4,0 \
  inplane_ws:32,7,4,2,3,1,4,0 inplane_ws:32,7,4,2,4,1,4,0 \
  inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:16,16,4,4,6,2,1,0 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:16,16,4,4,4,2,2,9 \
  > gpurun_out/ws3_ab.json 2> gpurun_out/ws3_ab.err
cat gpurun_out/ws3_ab.json
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --tune none"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:inplane_ws -s 4 -c 1 -o gpurun_out/ws3_ry4 $B --iters 6 --kernel inplane_ws --config 16,16,4,4,4,2,2,0 > gpurun_out/ncu_ws3_ry4.log 2>&1
