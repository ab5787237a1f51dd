#!/bin/bash
# round 2: tune both in-plane kernels + forward + c5 on the box (fills tune_cache.txt), then the
# cached bench twice; tune_cache.txt comes back in gpurun_out
set -x
rm -f tune_cache.txt
timeout 1500 python bench.py --steps 20 --warmup 3 > gpurun_out/b1_tune.json 2> gpurun_out/b1_tune.log
cp tune_cache.txt gpurun_out/tune_cache.txt
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/b1_cached.json 2> gpurun_out/b1_cached.log
cat gpurun_out/b1_cached.json
