# A/B: tools/variants/old.so (0b5f654) vs the current in-tree build
cp paper_conf_ipps_tangtkwkgtw13_b200/libstencil.so tools/variants/new.so
CFGS="${CFGS:-32,8,4,4,4,2,2,0 16,16,4,4,4,1,2,0,148 32,8,4,4,4,1,2,0,148 16,16,4,2,4,1,4,0,296 32,8,4,2,4,1,2,0,296}" ITERS="${ITERS:-4 100}" VARS="${VARS:-old new}" bash tools/abv.sh
