#!/bin/bash
# A/B: tools/variants/v1old.so vs the in-tree build on the classic in-plane kernel
set -x
timeout 120 python -m pytest tests/test_parity_gpu.py -x -q --timeout 60 -k "random_field_10 and inplane" > gpurun_out/abv1_tests.log 2>&1; tail -2 gpurun_out/abv1_tests.log
gunzip -k -f tools/variants/v1old.so.gz
C="inplane:16,16,4,4,4,2,2,0 inplane:32,8,4,4,4,2,2,0 inplane:16,15,4,4,4,2,2,0 inplane:32,7,4,2,4,1,4,0"
for i in 1 2 3; do
  STENCIL_LIB=tools/variants/v1old.so timeout 200 python tools/ab_configs.py --rounds 4 $C > gpurun_out/abv1_old_$i.json 2>/dev/null
  timeout 200 python tools/ab_configs.py --rounds 4 $C > gpurun_out/abv1_new_$i.json 2>/dev/null
done
