#!/bin/bash
set -x
timeout 900 python -m pytest tests/test_p2p_gpu.py tests/test_tune_gpu.py tests/test_run_until_gpu.py -v -m gpu --timeout 200 > gpurun_out/t2.log 2>&1
grep -E "PASSED|FAILED|ERROR" gpurun_out/t2.log | grep -v PASSED; tail -2 gpurun_out/t2.log
