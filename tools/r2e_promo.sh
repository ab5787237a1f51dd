#!/bin/bash
# TMA L2 promotion of the plane boxes (STENCIL_L2_PROMO): 128 B (default) vs 64 B vs none -- DRAM bytes per sweep
# and the sustained rate (the pitched rows' shell lines are fetched whole under 128-B promotion)
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,6,2,1,0"
for i in 1 2; do
  for P in 128 64 none; do
    STENCIL_L2_PROMO=$P timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/promo_sus_$P.jsonl 2>>gpurun_out/promo.err
  done
done
for P in 128 64 none; do
  STENCIL_L2_PROMO=$P timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum --cache-control none --clock-control none -k regex:inplane -s 3 -c 3 --csv python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 8 inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/promo_ncu_$P.csv 2>/dev/null
  STENCIL_L2_PROMO=$P timeout 300 python tools/sustained_ab.py --r 4 --dtype f64 --seconds 1.0 --rounds 2 inplane_ws:16,16,2,4,6,1,1,0 >> gpurun_out/promo_f64_$P.jsonl 2>>gpurun_out/promo.err
  STENCIL_L2_PROMO=$P timeout 300 python tools/sustained_ab.py --r 1 --seconds 1.0 --rounds 2 inplane_ws:32,4,4,4,4,1,2,0 >> gpurun_out/promo_r1_$P.jsonl 2>>gpurun_out/promo.err
done
