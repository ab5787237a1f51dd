// kern_f64_r2_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r2_ws, double, 2, false)
