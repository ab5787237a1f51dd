#!/bin/bash
# Final pass after the 64-B L2 promotion default: GPU suite, smoke, profiling pass (TAG=r2f), bench lines, and a
# second-box confirmation of the promotion A/B
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2f_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r2f_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2f_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2f_smoke.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2f_bench1.json 2> gpurun_out/r2f_bench1.err
TAG=r2f bash tools/profile_r2.sh > gpurun_out/prof_r2f.log 2>&1
C="inplane_ws:32,8,4,4,4,2,2,0"
for i in 1 2; do
  for P in 128 64; do
    STENCIL_L2_PROMO=$P timeout 300 python tools/sustained_ab.py --seconds 1.0 --rounds 2 $C >> gpurun_out/r2f_promo_$P.jsonl 2>>gpurun_out/r2f_promo.err
  done
done
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/r2f_bench2.json 2> gpurun_out/r2f_bench2.err
