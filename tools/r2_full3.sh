#!/bin/bash
set -x
start=$(date +%s)
timeout 3000 python -m pytest tests -q -m gpu --timeout 600 -x > gpurun_out/gputest_full3.log 2>&1; echo "rc=$? secs=$(( $(date +%s) - start ))" >> gpurun_out/gputest_full3.log
tail -4 gpurun_out/gputest_full3.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke3.log 2>&1; tail -4 gpurun_out/smoke3.log
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench3.json 2> gpurun_out/bench3.log; cat gpurun_out/bench3.json | head -c 400
