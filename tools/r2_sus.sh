#!/bin/bash
set -x
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:16,16,4,4,4,2,2,0 inplane_ws:16,16,4,2,4,1,2,0 inplane_ws:16,16,4,2,6,1,2,0 inplane_ws:32,7,4,2,3,1,4,0 inplane_ws:32,8,4,2,4,1,4,0 inplane:16,16,4,4,4,2,2,0 inplane:16,15,4,4,4,2,2,0"
timeout 900 python tools/sustained_ab.py --seconds 1.0 --rounds 3 $C > gpurun_out/sus1.json 2> gpurun_out/sus1.err
B="python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 6"
for c in $C; do
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --cache-control none --clock-control none -k regex:inplane -s 2 -c 3 --csv $B $c > gpurun_out/dram_$(echo $c | tr ':,' '__').csv 2>/dev/null
done
ls gpurun_out | grep dram_ | head
