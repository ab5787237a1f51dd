#!/bin/bash
# round 2: first GPU pass of the warp-specialized in-plane kernel (every step under its own timeout)
set -x
timeout 60 python tools/ws_smoke.py > gpurun_out/ws1_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/ws1_smoke.log
cat gpurun_out/ws1_smoke.log
grep -q "bit-identical to inplane: True" gpurun_out/ws1_smoke.log || exit 1
timeout 600 python -m pytest tests/test_parity_gpu.py -x -q --timeout 120 -k "random_field or integer_field or wide" > gpurun_out/ws1_tests.log 2>&1
tail -5 gpurun_out/ws1_tests.log
timeout 300 python tools/tune_one.py --kernel inplane_ws --dtype f32 --top 30 > gpurun_out/ws1_tune.log 2>&1
head -12 gpurun_out/ws1_tune.log
timeout 400 python tools/ab_configs.py --rounds 5 \
  inplane:16,16,4,4,4,2,2,0 inplane:16,15,4,4,6,2,1,0 inplane:32,7,4,2,4,1,4,0 \
  inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:16,16,4,4,6,2,1,0 inplane_ws:16,16,4,4,3,2,4,0 inplane_ws:16,16,4,4,4,2,2,9 \
  inplane_ws:32,7,4,2,4,1,4,0 inplane_ws:32,7,4,2,6,1,2,0 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:16,8,4,4,6,4,2,0 \
  > gpurun_out/ws1_ab.json 2> gpurun_out/ws1_ab.err
cat gpurun_out/ws1_ab.json
