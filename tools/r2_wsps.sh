#!/bin/bash
# warp-specialized fused peer-store slabs: parity, then tune-cache entries for the C5 p2p slabs
set -x
timeout 1200 python -m pytest tests/test_p2p_gpu.py -q -m gpu --timeout 600 -x > gpurun_out/wsps_tests.log 2>&1; tail -3 gpurun_out/wsps_tests.log
cp tune_cache.txt gpurun_out/tune_cache_before.txt
timeout 1500 python tools/tune_c5_slabs.py > gpurun_out/wsps_tune.log 2>&1; tail -12 gpurun_out/wsps_tune.log
cp tune_cache.txt gpurun_out/tune_cache_after.txt
