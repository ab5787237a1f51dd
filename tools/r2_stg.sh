#!/bin/bash
# A/B: v2.f32 / v4.f32 output stores (libstencil.so) vs the u64 operand form ($PWD/ab_variants/stg_u64.so)
C="inplane_ws:32,8,4,4,4,2,2,0 inplane:16,15,4,4,4,2,2,0"
for i in 1 2; do
  for v in base u64; do
    if [ $v = base ]; then L=""; else L=$PWD/ab_variants/stg_u64.so; fi
    STENCIL_LIB=$L timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 3 $C > gpurun_out/stg_${v}_$i.json 2> gpurun_out/stg_${v}_$i.err
  done
done
for v in base u64; do
  if [ $v = base ]; then L=""; else L=$PWD/ab_variants/stg_u64.so; fi
  STENCIL_LIB=$L timeout 300 python bench.py --steps 20 --warmup 3 > gpurun_out/stg_bench_$v.json 2> gpurun_out/stg_bench_$v.err
  STENCIL_LIB=$L timeout 300 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:inplane -s 2 -c 4 --csv python tools/run_config.py --n 512 --nz 512 --r 4 --dtype f32 --iters 6 inplane_ws:32,8,4,4,4,2,2,0 > gpurun_out/stg_ncu_$v.csv 2>/dev/null
done

