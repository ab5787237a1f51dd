python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$? >> gpurun_out/pytest_gpu.log
for i in 1 2; do timeout 600 python bench.py > gpurun_out/bench_default_$i.json 2> gpurun_out/bench_default_$i.err; done
