#!/bin/bash
set -x
for f in test_dist_local_gpu test_tune_gpu test_p2p_gpu test_parity_gpu; do
  timeout 900 python -m pytest tests/$f.py -v -m gpu --timeout 300 -x > gpurun_out/t1_$f.log 2>&1
  tail -3 gpurun_out/t1_$f.log
done
