#!/bin/bash
# classic in-plane kernel (K-IP): 16-byte v4.f32 output stores (default) vs two 8-byte lane stores (-DSTENCIL_STG64)
V=$PWD/ab_variants/c64.so
for i in 1 2; do
  for L in "" $V; do
    T=$([ -z "$L" ] && echo base || echo c64)
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r 4 --seconds 1.0 --rounds 2 inplane:16,15,4,4,4,2,2,0 inplane:32,8,4,4,4,2,2,0 >> gpurun_out/c64_r4_$T.jsonl 2>>gpurun_out/c64.err
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r 2 --seconds 1.0 --rounds 2 inplane:16,16,4,2,6,1,2,0 >> gpurun_out/c64_r2_$T.jsonl 2>>gpurun_out/c64.err
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r 1 --seconds 1.0 --rounds 2 inplane:16,8,4,4,6,1,1,0 >> gpurun_out/c64_r1_$T.jsonl 2>>gpurun_out/c64.err
  done
done
