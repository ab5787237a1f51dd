#!/bin/bash
# Final round-2 GPU pass on the committed build: GPU suite, smoke, two bench lines, C1/C3 + Div/Grad
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/fin_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/fin_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fin_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/fin_smoke.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/fin_bench1.json 2> gpurun_out/fin_bench1.err
export STENCIL_TUNE_SUSTAIN_MS=150
timeout 2400 python tools/configs_bench.py > gpurun_out/configs_r2d.json 2> gpurun_out/configs_r2d.log
timeout 1500 python tools/divgrad_bench.py > gpurun_out/divgrad_r2d.json 2> gpurun_out/divgrad_r2d.log
unset STENCIL_TUNE_SUSTAIN_MS
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/fin_bench2.json 2> gpurun_out/fin_bench2.err
