// kern_f64_r1_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r1_ws, double, 1, false)
