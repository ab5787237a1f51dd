#!/bin/bash
# Final round-2 validation on the built library: GPU suite, smoke, memcheck of the kernels whose stores changed,
# and a default bench line
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/val_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/val_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/val_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/val_smoke.log
for c in ws_f32_r4 ip_f32_r4 ps_ws_f32_r2 ps_ip_f32_r2; do
  timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python tools/sanitize_case.py $c > gpurun_out/val_memcheck_$c.log 2>&1
  echo "rc=$?" >> gpurun_out/val_memcheck_$c.log
done
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/val_bench.json 2> gpurun_out/val_bench.err
