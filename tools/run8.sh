python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
(python paper_conf_ipps_tangtkwkgtw13_b200/build.py --force --out tools/variants/split.so -D STENCIL_ISO_SPLIT=1 > gpurun_out/build_split.log 2>&1) &
BPID=$!
timeout 600 python -m pytest tests/test_graphs_gpu.py tests/test_parity_gpu.py -q -x > gpurun_out/pytest_graphs.log 2>&1; echo rc=$? >> gpurun_out/pytest_graphs.log
timeout 600 python tools/c1_bench.py > gpurun_out/c1.json 2> gpurun_out/c1.err
wait $BPID
rm -f gpurun_out/abv.txt
CFGS="16,15,4,4,4,2,2,0 32,8,4,4,4,2,2,0 32,7,4,2,4,1,4,0" ITERS="4 100" VARS="new split" bash tools/ab1.sh
