python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$? >> gpurun_out/pytest_gpu.log
for c in ${CFGS:-16,16,4,4,4,2,2,0 16,15,4,4,4,2,2,0 32,8,4,4,4,2,2,0 16,8,4,4,4,2,2,0}; do for it in ${ITERS:-4 100}; do
    echo "cfg=$c iters=$it" >> gpurun_out/quick.txt
    timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --iters $it --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_ms'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" >> gpurun_out/quick.txt
done; done
