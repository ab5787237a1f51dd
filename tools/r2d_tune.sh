#!/bin/bash
# Exhaustive re-tune of C2 on the final kernels (appends the winners to tune_cache.txt), the profiling pass of
# whatever tuple bench.py then times (TAG=r2d), and a bench line
timeout 2400 python bench.py --tune exhaustive --steps 20 --warmup 3 > gpurun_out/tune_bench.json 2> gpurun_out/tune_bench.err
cp tune_cache.txt gpurun_out/tune_cache_new.txt
TAG=r2d bash tools/profile_r2.sh > gpurun_out/prof_r2d.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_after_tune.json 2> gpurun_out/bench_after_tune.err
