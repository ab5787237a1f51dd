# profiling pass for the current kernel: launch list + ncu full of two near-equal tuned configs
CFG=16,15,4,4,4,2,2,0 TAG=r1e bash tools/profile.sh
B="python bench.py --profile --steps 2 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --tune none"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:inplane_sweep -s 4 -c 1 -o gpurun_out/inplane_r1e2 $B --iters 6 --config 32,8,4,4,4,2,2,0 > gpurun_out/ncu_full_ip2.log 2>&1
ls gpurun_out
