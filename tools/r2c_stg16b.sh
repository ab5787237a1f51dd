#!/bin/bash
# A/B of the store-width rule (inplane_ws.cuh STG16 = fp64 || r >= 5) on cases the first A/B did not cover:
# the default build against variants with the opposite width forced (ab_variants/v8.so: fp32 r5, fp64 r2, r6
# with 8-byte stores; ab_variants/v16.so: fp32 r2, r3 with 16-byte stores)
ab() {  # variant dtype r cfg
  for i in 1 2; do
    for L in "" $PWD/ab_variants/$1.so; do
      T=$([ -z "$L" ] && echo base || echo $1)
      STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r $3 --dtype $2 --seconds 1.0 --rounds 2 $4 >> gpurun_out/stg16b_$2r$3_$T.jsonl 2>>gpurun_out/stg16b.err
    done
  done
}
ab v8 f32 5 inplane_ws:32,7,4,2,4,1,2,0
ab v8 f64 2 inplane_ws:32,8,2,4,3,1,2,0
ab v8 f64 6 inplane_ws:32,7,2,2,4,1,2,0
ab v16 f32 3 inplane_ws:32,8,4,2,6,1,2,0
ab v16 f32 2 inplane_ws:32,8,4,2,6,1,2,0
