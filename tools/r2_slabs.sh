#!/bin/bash
set -x
cp tune_cache.txt gpurun_out/tune_cache_before.txt
timeout 1500 python tools/tune_c5_slabs.py > gpurun_out/slabs.log 2>&1; tail -12 gpurun_out/slabs.log
cp tune_cache.txt gpurun_out/tune_cache_slabs.txt
