#!/bin/bash
# L2 eviction-priority hints, the pairs tools/r2_pol.sh did not cover: outputs evict_last (2) with inputs
# normal (0) / evict_first (1), against the default (0 0).  Sustained A/B + DRAM bytes across sweeps.
C="inplane_ws:32,8,4,4,4,2,2,0"
B="python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 8"
for pol in "0 0" "2 0" "2 1" "0 0" "2 1"; do set -- $pol
  export STENCIL_STORE_POLICY=$1 STENCIL_LOAD_POLICY=$2
  timeout 600 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/pol2_$1$2.json 2>/dev/null
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --cache-control none --clock-control none -k regex:inplane -s 3 -c 4 --csv $B $C > gpurun_out/pol2_dram_$1$2.csv 2>/dev/null
done
