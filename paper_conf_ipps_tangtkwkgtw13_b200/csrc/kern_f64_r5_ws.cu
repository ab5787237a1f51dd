// kern_f64_r5_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r5_ws, double, 5, false)
