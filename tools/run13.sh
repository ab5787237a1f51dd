python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python bench.py --workload c5 --tune beta5 --steps 3 --warmup 3 --iters 20 --no-cpu > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
