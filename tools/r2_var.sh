#!/bin/bash
# A/B of compile-time variants of the warp-specialized kernel, built on the box (the library is too large
# to ship several copies): base, stores without "memory" clobber, plain C++ shared loads, both
set -x
nproc
B="from paper_conf_ipps_tangtkwkgtw13_b200 import build as b; import sys; b.build(force=True, defines=sys.argv[2:], out=sys.argv[1])"
start=$(date +%s)
timeout 900 python -c "$B" /tmp/v_nc.so STENCIL_STG_NOCLOBBER > gpurun_out/var_build.log 2>&1
timeout 900 python -c "$B" /tmp/v_lp.so STENCIL_LDS_PLAIN >> gpurun_out/var_build.log 2>&1
timeout 900 python -c "$B" /tmp/v_both.so STENCIL_STG_NOCLOBBER STENCIL_LDS_PLAIN >> gpurun_out/var_build.log 2>&1
echo "build secs $(( $(date +%s) - start ))"; ls -la /tmp/v_*.so
ab() {  # tag dtype r cfgs...
  local tag=$1 dt=$2 r=$3; shift 3
  for i in 1 2; do
    for v in base nc lp both; do
      if [ $v = base ]; then L=""; else L=/tmp/v_$v.so; fi
      STENCIL_LIB=$L timeout 300 python tools/ab_configs.py --r $r --dtype $dt --rounds 3 "$@" > gpurun_out/var_${tag}_${v}_$i.json 2>gpurun_out/var_${tag}_${v}_$i.err
    done
  done
}
ab f32r4 f32 4 inplane_ws:32,8,4,4,4,2,2,0 inplane_ws:16,16,4,4,6,2,1,0
ab f32r6 f32 6 inplane_ws:32,7,4,2,6,1,1,0 inplane_ws:32,7,4,2,4,1,2,0
ab f64r4 f64 4 inplane_ws:32,8,2,4,6,1,1,0 inplane_ws:32,8,2,4,4,1,2,0
ab f64r6 f64 6 inplane_ws:32,7,2,2,3,1,2,0
