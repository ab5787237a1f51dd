#!/bin/bash
# (The STENCIL_LOCKSTEP hook was an experiment build, not kept in the tree; results in profiles/r2c/lockstep/.)
# Experiment: K-IP/WS lockstep between y-neighbour CTAs (STENCIL_LOCKSTEP = allowed drift in TMA loads)
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,6,2,1,0"
for i in 1 2; do
  for D in 0 1 2 4 8; do
    if [ $D = 0 ]; then unset STENCIL_LOCKSTEP; else export STENCIL_LOCKSTEP=$D; fi
    timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/lock_sus_$D.jsonl 2>>gpurun_out/lock.err
  done
done
for D in 0 2 4; do
  if [ $D = 0 ]; then unset STENCIL_LOCKSTEP; else export STENCIL_LOCKSTEP=$D; fi
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_op_read_hit_rate.pct --cache-control none --clock-control none -k regex:inplane -s 3 -c 3 --csv python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 8 inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/lock_ncu_$D.csv 2>/dev/null
done
unset STENCIL_LOCKSTEP
