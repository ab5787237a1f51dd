#!/bin/bash
# Exhaustive re-tune of C2 with the widened sustained refinement (twelve fastest + four fastest of the largest
# register tiles, 1 s runs), replacing the C2 tune-cache lines measured on earlier kernels; then the profiling
# pass of the new timed tuple (TAG=r2e) and two bench lines
export STENCIL_TUNE_SUSTAIN_MS=1000
timeout 3000 python bench.py --tune exhaustive --steps 20 --warmup 3 > gpurun_out/r2e_tune_bench.json 2> gpurun_out/r2e_tune_bench.err
unset STENCIL_TUNE_SUSTAIN_MS
cp tune_cache.txt gpurun_out/tune_cache_r2e.txt
TAG=r2e bash tools/profile_r2.sh > gpurun_out/prof_r2e.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2e_bench1.json 2> gpurun_out/r2e_bench1.err
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2e_bench2.json 2> gpurun_out/r2e_bench2.err
