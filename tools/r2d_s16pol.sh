#!/bin/bash
# f32 r=4: 16-byte stores with an L2 evict_first hint on the outputs vs the default 8-byte stores; then the GPU suite
V=$PWD/ab_variants/s16r4.so
C="inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,6,2,1,0"
for i in 1 2; do
  timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/s16pol_base.jsonl 2>>gpurun_out/s16pol.err
  STENCIL_LIB=$V timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/s16pol_s16.jsonl 2>>gpurun_out/s16pol.err
  STENCIL_STORE_POLICY=1 STENCIL_LIB=$V timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/s16pol_s16ef.jsonl 2>>gpurun_out/s16pol.err
done
for T in base s16ef; do
  if [ $T = base ]; then L=""; P=0; else L=$V; P=1; fi
  STENCIL_STORE_POLICY=$P STENCIL_LIB=$L timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none -k regex:inplane -s 3 -c 3 --csv python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 8 inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/s16pol_ncu_$T.csv 2>/dev/null
done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/fin2_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/fin2_gputest.log
