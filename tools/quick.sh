python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$? >> gpurun_out/pytest_gpu.log
for c in 16,15,4,4,4,2,2,0 16,16,4,4,4,2,2,9 32,8,4,4,4,2,2,0; do for it in 4 100; do
    echo "cfg=$c iters=$it" >> gpurun_out/quick.txt
    timeout 120 python bench.py --steps 5 --warmup 3 --tune none --config $c --iters $it --no-cpu --no-e2e --no-baseline-kernel 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_ms'], d['clocks'])" >> gpurun_out/quick.txt
done; done
timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:inplane_sweep -s 3 -c 4 python bench.py --profile --iters 6 --steps 1 --warmup 1 --no-e2e --no-cpu --no-baseline-kernel --config 16,15,4,4,4,2,2,0 > gpurun_out/ncu_dir.txt 2>&1
