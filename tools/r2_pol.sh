#!/bin/bash
# L2 eviction-priority hints for the sweep's stores / TMA loads: sustained A/B + DRAM bytes
set -x
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,7,4,2,3,1,4,0 inplane_ws:16,16,4,4,4,2,2,0"
B="python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 6"
for pol in "0 0" "1 0" "0 1" "1 1" "0 2"; do set -- $pol
  export STENCIL_STORE_POLICY=$1 STENCIL_LOAD_POLICY=$2
  timeout 600 python tools/sustained_ab.py --seconds 0.7 --rounds 2 $C > gpurun_out/pol_$1$2.json 2>/dev/null
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none -k regex:inplane -s 2 -c 3 --csv $B inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/pol_dram_$1$2.csv 2>/dev/null
done
