#!/bin/bash
# A/B: 16-byte output stores (libstencil.so) vs per-lane 8-byte stores (ab_variants/stg8.so, -DSTENCIL_STG8)
V=$PWD/ab_variants/stg8.so
for i in 1 2; do
  for L in "" $V; do
    T=$([ -z "$L" ] && echo base || echo stg8)
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:32,8,4,4,6,2,1,0 >> gpurun_out/stg16_f32r4_$T.jsonl 2>>gpurun_out/stg16.err
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r 6 --seconds 1.0 --rounds 2 inplane_ws:32,7,4,2,3,1,4,0 >> gpurun_out/stg16_f32r6_$T.jsonl 2>>gpurun_out/stg16.err
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --r 4 --dtype f64 --seconds 1.0 --rounds 2 inplane_ws:16,16,2,4,3,1,2,0 >> gpurun_out/stg16_f64r4_$T.jsonl 2>>gpurun_out/stg16.err
    STENCIL_LIB=$L timeout 300 python tools/dg_ab.py grad f32 4 32,4,4,4,3,1,2 >> gpurun_out/stg16_dg_$T.jsonl 2>>gpurun_out/stg16.err
    STENCIL_LIB=$L timeout 300 python tools/dg_ab.py grad f64 4 32,8,2,4,2,1,2 >> gpurun_out/stg16_dg_$T.jsonl 2>>gpurun_out/stg16.err
  done
done
for L in "" $V; do
  T=$([ -z "$L" ] && echo base || echo stg8)
  STENCIL_LIB=$L timeout 300 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:inplane -s 2 -c 2 --csv python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 5 inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/stg16_ncu_$T.csv 2>/dev/null
done
