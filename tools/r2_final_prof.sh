#!/bin/bash
# After the store change: sustained A/B of the leading tuples, the profiling pass (TAG=r2c) and a bench line
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,3,2,2,0 inplane_ws:32,8,4,4,6,2,1,0 inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:32,7,4,2,3,1,4,0 inplane:16,15,4,4,4,2,2,0"
timeout 900 python tools/sustained_ab.py --seconds 1.0 --rounds 3 $C > gpurun_out/sus_r2c.json 2> gpurun_out/sus_r2c.err
TAG=r2c bash tools/profile_r2.sh > gpurun_out/prof_r2c.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_r2c.json 2> gpurun_out/bench_r2c.err
