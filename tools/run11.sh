python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$? >> gpurun_out/pytest_gpu.log
(cd tools/variants/basepkg && python paper_conf_ipps_tangtkwkgtw13_b200/build.py --force --out ../base.so > ../../../gpurun_out/build_base.log 2>&1)
rm -f gpurun_out/abv.txt
CFGS="16,16,4,4,4,2,2,0 16,15,4,4,4,2,2,0 16,16,4,4,4,1,2,0,148 32,8,4,4,4,1,2,0,148 16,8,4,4,4,1,2,0,296 16,8,4,4,6,1,1,0,296 32,7,4,2,4,1,4,0,148" ITERS="4 100" VARS="base new" bash tools/ab1.sh
