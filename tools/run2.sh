python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$? >> gpurun_out/pytest_gpu.log
CFGS="32,8,4,4,4,2,2,0 16,15,4,4,4,2,2,0" ITERS="4 100" bash tools/ab1.sh
