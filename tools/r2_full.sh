#!/bin/bash
set -x
timeout 2400 python -m pytest tests -x -q -m gpu --timeout 600 > gpurun_out/gputest_full.log 2>&1; tail -5 gpurun_out/gputest_full.log
TAG=r2a bash tools/profile_r2.sh
