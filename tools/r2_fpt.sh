#!/bin/bash
# forward-plane + TMA: parity, then the loading ablation again with the new row, and its ncu metrics
set -x
timeout 900 python -m pytest tests/test_parity_gpu.py -q -m gpu --timeout 300 -x -k "fp_tma or loading_variants" > gpurun_out/fpt_tests.log 2>&1; tail -3 gpurun_out/fpt_tests.log
timeout 1800 python tools/ablation.py > gpurun_out/ablation.json 2> gpurun_out/ablation.log
tail -3 gpurun_out/ablation.log
timeout 1200 python tools/ablation_ncu.py gpurun_out/ablation.json --r 4 > gpurun_out/ablation_ncu_r4.json 2> gpurun_out/ablation_ncu_r4.log
timeout 900 python tools/ablation_ncu.py gpurun_out/ablation.json --r 1 > gpurun_out/ablation_ncu_r1.json 2> gpurun_out/ablation_ncu_r1.log
