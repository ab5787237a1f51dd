#!/bin/bash
# round 2 baseline: driver-style bench + ncu source profile of the bench's config
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > gpurun_out/smi.txt
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_base.json 2> gpurun_out/bench_base.log
CFG=$(python -c "import json;d=json.load(open('gpurun_out/bench_base.json'));c=d['config']['kernel'];print(','.join(str(c[k]) for k in ['tx','ty','rx','ry','stages','zsegs','zbox','ytiles']))")
echo $CFG > gpurun_out/base_cfg.txt
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --tune none"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:inplane_sweep -s 4 -c 1 -o gpurun_out/ip_base $B --iters 6 --config $CFG > gpurun_out/ncu_base.log 2>&1
ls -la gpurun_out
