#!/bin/bash
# C1 / C3 (configs_bench.py) and Div / Grad on the kernels with in-place stores
export STENCIL_TUNE_SUSTAIN_MS=150
timeout 2400 python tools/configs_bench.py > gpurun_out/configs_r2c.json 2> gpurun_out/configs_r2c.log; tail -3 gpurun_out/configs_r2c.log
timeout 1500 python tools/divgrad_bench.py > gpurun_out/divgrad_r2c.json 2> gpurun_out/divgrad_r2c.log; tail -3 gpurun_out/divgrad_r2c.log
