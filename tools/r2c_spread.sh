#!/bin/bash
# Experiment (round 2, not adopted): spread the 20 idle SMs of the 128-CTA grid over the machine
# (STENCIL_SPREAD=keep,per). The hook was an uncommitted experiment build (a 1-D grid remap in inplane_ws.cuh
# and the launch in plan.cu), not kept in the tree; results in profiles/r2c/spread/
L=$PWD/ab_variants/spread.so
C=inplane_ws:32,8,4,4,4,2,2,0
for i in 1 2; do
  STENCIL_LIB=$L timeout 300 python tools/ts_gaps.py $C >> gpurun_out/spread_ts_base.jsonl 2>>gpurun_out/spread.err
  STENCIL_SPREAD=32,37 STENCIL_LIB=$L timeout 300 python tools/ts_gaps.py $C >> gpurun_out/spread_ts_s3237.jsonl 2>>gpurun_out/spread.err
  STENCIL_SPREAD=8,9 STENCIL_LIB=$L timeout 300 python tools/ts_gaps.py $C >> gpurun_out/spread_ts_s89.jsonl 2>>gpurun_out/spread.err
done
for i in 1 2; do
  STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --seconds 1.5 --rounds 2 $C >> gpurun_out/spread_sus_base.jsonl 2>>gpurun_out/spread.err
  STENCIL_SPREAD=32,37 STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --seconds 1.5 --rounds 2 $C >> gpurun_out/spread_sus_s3237.jsonl 2>>gpurun_out/spread.err
  STENCIL_SPREAD=8,9 STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --seconds 1.5 --rounds 2 $C >> gpurun_out/spread_sus_s89.jsonl 2>>gpurun_out/spread.err
done
