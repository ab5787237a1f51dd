python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for promo in 128 none 256; do
  for c in 16,16,4,4,4,2,2 32,8,4,4,4,2,2 32,7,4,2,4,1,4 16,8,4,4,4,2,2; do
    echo "promo=$promo cfg=$c" >> gpurun_out/quick.txt
    STENCIL_L2_PROMO=$promo timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_ms'], d['clocks']['sm_mhz'])" >> gpurun_out/quick.txt
  done
done
