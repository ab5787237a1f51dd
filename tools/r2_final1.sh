#!/bin/bash
set -x
start=$(date +%s)
timeout 3000 python -m pytest tests -q -m gpu --timeout 600 -x > gpurun_out/gputest_f1.log 2>&1; echo "rc=$? secs=$(( $(date +%s) - start ))" >> gpurun_out/gputest_f1.log
tail -4 gpurun_out/gputest_f1.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_f1.log 2>&1; tail -4 gpurun_out/smoke_f1.log
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_f1.json 2> gpurun_out/bench_f1.log; head -c 300 gpurun_out/bench_f1.json
timeout 2400 python tools/configs_bench.py --c4-only > gpurun_out/c4_r2.json 2> gpurun_out/c4_r2.log; tail -3 gpurun_out/c4_r2.log
