#!/bin/bash
set -x
timeout 600 python -m pytest tests/test_parity_gpu.py -x -q --timeout 120 -k "random_field or integer_field or wide" > gpurun_out/ws2_tests.log 2>&1
tail -3 gpurun_out/ws2_tests.log
timeout 400 python tools/ab_configs.py --rounds 6 \
  inplane:16,16,4,4,4,2,2,0 inplane:16,15,4,4,6,2,1,0 inplane:32,7,4,2,4,1,4,0 \
  inplane_ws:32,7,4,2,3,1,4,0 inplane_ws:16,16,4,2,6,1,2,0 inplane_ws:32,7,4,2,4,1,4,0 \
  inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:16,16,4,4,6,2,1,0 inplane_ws:32,8,4,4,4,2,2,0 \
  > gpurun_out/ws2_ab.json 2> gpurun_out/ws2_ab.err
cat gpurun_out/ws2_ab.json
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --tune none"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:inplane_ws -s 4 -c 1 -o gpurun_out/ws_ry2 $B --iters 6 --kernel inplane_ws --config 32,7,4,2,3,1,4,0 > gpurun_out/ncu_ws_ry2.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:inplane_ws -s 4 -c 1 -o gpurun_out/ws_ry4 $B --iters 6 --kernel inplane_ws --config 16,16,4,4,4,2,2,0 > gpurun_out/ncu_ws_ry4.log 2>&1
ls gpurun_out
