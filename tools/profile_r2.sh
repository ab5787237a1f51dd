#!/bin/bash
# Round-2 profiling pass of the configuration bench.py times (tune_cache.txt), run under gpurun:
#   launch list of a short bench run, ncu --set full of the in-plane sweep (exact timed config) and of
#   the forward-plane baseline, DRAM bytes without cache flushes.  tools/ncu_summary.py -> profiles/.
set -x
TAG=${TAG:-r2}
CFGJ=$(python -c "import bench;c=bench.pinned_config('c2');print(c['kernel']+':'+','.join(str(c[k]) for k in bench.KEYS))")
K=${CFGJ%%:*}; CFG=${CFGJ#*:}
FCFG=$(python -c "import bench;e=bench.cache_entry(512,512,512,4,'f32',kernel='forward');print(','.join(str(e[1][k]) for k in bench.KEYS))")
echo "$CFGJ" > gpurun_out/profile_cfg_$TAG.txt
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --no-c5 --tune none"
KRE=$([ "$K" = inplane_ws ] && echo inplane_ws_kernel || echo inplane_sweep)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv $B --iters 10 --kernel $K --config $CFG > gpurun_out/ncu_launches_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$KRE -s 4 -c 1 -o gpurun_out/inplane_$TAG $B --iters 6 --kernel $K --config $CFG > gpurun_out/ncu_full_ip_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:forward_sweep -s 2 -c 1 -o gpurun_out/forward_$TAG $B --iters 3 --kernel forward --config $FCFG > gpurun_out/ncu_full_fp_$TAG.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --cache-control none --clock-control none -k regex:$KRE -s 4 -c 4 --csv --log-file gpurun_out/dram_nocacheflush_$TAG.csv $B --iters 10 --kernel $K --config $CFG > gpurun_out/ncu_dram_$TAG.log 2>&1
ls -la gpurun_out
