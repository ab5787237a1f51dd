python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in "f32 1" "f64 4"; do set -- $c
  CFGJ=$(python tools/ncu_case.py $1 $2 --tune 2> gpurun_out/ncu_$1_r$2.tune.err | tail -1)
  echo "$CFGJ" > gpurun_out/ncu_$1_r$2.cfg
  timeout 900 ncu --set full --clock-control none -k regex:inplane_sweep -s 2 -c 1 -o gpurun_out/ncu_$1_r$2 python tools/ncu_case.py $1 $2 "$CFGJ" > gpurun_out/ncu_$1_r$2.log 2>&1 || true
done
ls gpurun_out
