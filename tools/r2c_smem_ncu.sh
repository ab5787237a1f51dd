#!/bin/bash
# Shared-memory crossbar load of the C3 configurations (profiles/r2c_rooflines.md): ncu metrics per sweep
M=gpu__time_duration.sum,sm__cycles_elapsed.avg.per_second,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__throughput.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
run() {  # tag dtype r json
  timeout 600 ncu --metrics $M --clock-control none -k regex:inplane -s 2 -c 1 --csv python tools/ncu_case.py $2 $3 "$4" > gpurun_out/smem_$1.csv 2> gpurun_out/smem_$1.err
}
run f32r4 f32 4 '{"kernel":"inplane_ws","tx":32,"ty":8,"rx":4,"ry":4,"stages":4,"zsegs":2,"zbox":2,"ytiles":0}'
run f32r5 f32 5 '{"kernel":"inplane_ws","tx":32,"ty":7,"rx":4,"ry":2,"stages":4,"zsegs":1,"zbox":2,"ytiles":0}'
run f32r6 f32 6 '{"kernel":"inplane_ws","tx":32,"ty":7,"rx":4,"ry":2,"stages":3,"zsegs":1,"zbox":4,"ytiles":0}'
run f64r4 f64 4 '{"kernel":"inplane_ws","tx":16,"ty":16,"rx":2,"ry":4,"stages":3,"zsegs":1,"zbox":2,"ytiles":0}'
run f64r5 f64 5 '{"kernel":"inplane_ws","tx":32,"ty":7,"rx":2,"ry":2,"stages":4,"zsegs":1,"zbox":2,"ytiles":0}'
run f64r6 f64 6 '{"kernel":"inplane_ws","tx":32,"ty":7,"rx":2,"ry":2,"stages":4,"zsegs":1,"zbox":2,"ytiles":0}'
