python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for sp in 0 1 2; do for lp in 0 1; do
  for c in 16,15,4,4,4,2,2,0; do
    echo "store=$sp load=$lp cfg=$c" >> gpurun_out/quick.txt
    STENCIL_STORE_POLICY=$sp STENCIL_LOAD_POLICY=$lp timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --iters 4 --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_ms'], d['clocks']['sm_mhz'])" >> gpurun_out/quick.txt
  done
done; done
STENCIL_STORE_POLICY=1 timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:inplane_sweep -s 3 -c 2 python bench.py --profile --iters 6 --steps 1 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --config 16,15,4,4,4,2,2,0 > gpurun_out/ncu_pol1.txt 2>&1
STENCIL_STORE_POLICY=0 timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:inplane_sweep -s 3 -c 2 python bench.py --profile --iters 6 --steps 1 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --config 16,15,4,4,4,2,2,0 > gpurun_out/ncu_pol0.txt 2>&1
