python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
mkdir -p tools/variants
python paper_conf_ipps_tangtkwkgtw13_b200/build.py --force --out tools/variants/stg64.so -D STENCIL_STG64 > gpurun_out/build_stg64.log 2>&1
rm -f gpurun_out/abv.txt
CFGS="16,16,4,4,4,2,2,0 32,8,4,4,4,2,2,18 16,15,4,4,4,2,2,0" ITERS="4 100" VARS="new stg64" bash tools/ab1.sh
