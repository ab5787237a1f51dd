#!/bin/bash
# Final pass with the per-grid L2 promotion rule: GPU suite, smoke, bench lines (c5_1gpu back at 128 B)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2g_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r2g_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2g_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2g_smoke.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2g_bench1.json 2> gpurun_out/r2g_bench1.err
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2g_bench2.json 2> gpurun_out/r2g_bench2.err
