#!/bin/bash
# Round profiling pass (run under gpurun from the repo root):
#   1. ncu launch list (gpu__time_duration of every kernel) of a short bench run
#   2. ncu --set full of the in-plane sweep and of the forward-plane baseline
# Reports land in gpurun_out/; tools/ncu_summary.py turns them into profiles/.
set -x
CFG=${CFG:-16,16,4,4,4,2,2,9}
FCFG=${FCFG:-16,4,1,1,1,1,1,0}
TAG=${TAG:-r1}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --tune none"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv $B --iters 10 --config $CFG > gpurun_out/ncu_launches.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:inplane_sweep -s 4 -c 1 -o gpurun_out/inplane_$TAG $B --iters 6 --config $CFG > gpurun_out/ncu_full_ip.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:forward_sweep -s 2 -c 1 -o gpurun_out/forward_$TAG $B --iters 3 --kernel forward --config $FCFG > gpurun_out/ncu_full_fp.log 2>&1
# cross-sweep L2 reuse needs the cache left alone between kernels
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --cache-control none --clock-control none -k regex:inplane_sweep -s 4 -c 4 --csv --log-file gpurun_out/dram_nocacheflush_$TAG.csv $B --iters 10 --config $CFG > gpurun_out/ncu_dram.log 2>&1
ls -la gpurun_out
