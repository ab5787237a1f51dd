#!/bin/bash
# A/B of prebuilt variants in tools/variants/*.so (one gpurun session).
for c in ${CFGS:-16,16,4,4,4,2,2,0}; do for it in ${ITERS:-4}; do for rep in 1 2; do for v in ${VARS:-old new}; do for e in ${ENVS:-X=0}; do
    r=$(env $e STENCIL_LIB=tools/variants/$v.so timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --iters $it --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['roofline']['avg_launch_ms'], d['clocks']['sm_mhz'], d['clocks']['reasons'])")
    echo "variant=$v env=$e cfg=$c iters=$it rep=$rep: $r" >> gpurun_out/abv.txt
done; done; done; done; done
