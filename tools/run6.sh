python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_p2p_gpu.py -q -x > gpurun_out/pytest_p2p.log 2>&1; echo rc=$? >> gpurun_out/pytest_p2p.log
