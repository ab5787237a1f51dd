#!/bin/bash
# A/B experiments in ONE gpurun session: build variants of libstencil.so with
# extra -D flags and time fixed configs with each (STENCIL_LIB selects the build).
# usage: VARIANTS="base: dbg:STENCIL_DEBUG_HOOKS" CFGS="..." ITERS="4" ENVS="STENCIL_DEBUG=0 STENCIL_DEBUG=3" bash tools/ab.sh
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
mkdir -p /tmp/variants
for v in ${VARIANTS:-base:}; do
  name=${v%%:*}; defs=${v#*:}
  args=""; for d in ${defs//,/ }; do args="$args -D $d"; done
  python paper_conf_ipps_tangtkwkgtw13_b200/build.py --force --out /tmp/variants/$name.so $args > /tmp/variants/$name.log 2>&1 || { echo "build $name failed" >> gpurun_out/ab.txt; cat /tmp/variants/$name.log >> gpurun_out/ab.txt; continue; }
  for e in ${ENVS:-X=0}; do for c in ${CFGS:-16,16,4,4,4,2,2,0}; do for it in ${ITERS:-4}; do
    r=$(env $e STENCIL_LIB=/tmp/variants/$name.so timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --iters $it --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['roofline']['avg_launch_ms'], d['clocks']['sm_mhz'], d['clocks']['reasons'])")
    echo "variant=$name env=$e cfg=$c iters=$it : $r" >> gpurun_out/ab.txt
  done; done; done
done
