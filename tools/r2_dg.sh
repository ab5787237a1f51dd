#!/bin/bash
set -x
timeout 900 python -m pytest tests/test_divgrad_gpu.py -v -m gpu --timeout 200 -x > gpurun_out/dg.log 2>&1
grep -E "FAILED|ERROR|passed|failed" gpurun_out/dg.log | head; grep -E "^E " gpurun_out/dg.log | head -20
