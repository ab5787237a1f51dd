python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2700 python tools/configs_bench.py --c4 > gpurun_out/configs_c4.json 2> gpurun_out/configs_c4.err
