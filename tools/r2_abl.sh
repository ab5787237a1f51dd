#!/bin/bash
set -x
timeout 1200 python -m pytest tests -q -m gpu --timeout 300 -x -k "tune_gpu or p2p" > gpurun_out/abl_tests.log 2>&1; tail -3 gpurun_out/abl_tests.log
timeout 1500 python tools/ablation.py > gpurun_out/ablation.json 2> gpurun_out/ablation.log
tail -3 gpurun_out/ablation.log
timeout 1200 python tools/ablation_ncu.py gpurun_out/ablation.json --r 4 > gpurun_out/ablation_ncu_r4.json 2> gpurun_out/ablation_ncu_r4.log
timeout 900 python tools/ablation_ncu.py gpurun_out/ablation.json --r 1 > gpurun_out/ablation_ncu_r1.json 2> gpurun_out/ablation_ncu_r1.log
