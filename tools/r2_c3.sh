#!/bin/bash
set -x
export STENCIL_TUNE_SUSTAIN_MS=150
timeout 1500 python tools/divgrad_bench.py > gpurun_out/divgrad.json 2> gpurun_out/divgrad.log; tail -3 gpurun_out/divgrad.log
timeout 2400 python tools/configs_bench.py > gpurun_out/configs_r2.json 2> gpurun_out/configs_r2.log; tail -3 gpurun_out/configs_r2.log
