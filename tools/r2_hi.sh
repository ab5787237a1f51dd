#!/bin/bash
# ncu --set full of the tuned high-order / fp64 sweeps (512^3), for the register / occupancy analysis
set -x
run() {  # name dtype r cfg
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"inplane|fp_tma" -s 2 -c 1 -f -o gpurun_out/hi_$1 \
    python tools/run_config.py --n 512 --nz 512 --r $3 --dtype $2 --iters 4 $4 > gpurun_out/hi_$1.log 2>&1
  ncu -i gpurun_out/hi_$1.ncu-rep --page raw --csv > gpurun_out/hi_$1_raw.csv 2>/dev/null
}
run f32r6 f32 6 inplane_ws:32,7,4,2,6,1,1,0
run f32r5 f32 5 inplane_ws:32,7,4,2,4,1,2,0
run f64r4 f64 4 inplane_ws:32,8,2,4,6,1,1,0
run f64r6 f64 6 inplane_ws:32,7,2,2,3,1,2,0
run f32r4 f32 4 inplane_ws:32,8,4,4,4,2,2,0
ls -la gpurun_out/ | grep hi_
