python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_p2p_gpu.py -q -k bench > gpurun_out/pytest_bench2.log 2>&1; echo rc=$? >> gpurun_out/pytest_bench2.log
STENCIL_BENCH_SAME_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --iters 10 --tune none --config 32,8,4,4,4,2,2,0 --no-cpu > gpurun_out/bench2.json 2> gpurun_out/bench2.err
