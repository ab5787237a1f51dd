// kern_f64_r3_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r3_ws, double, 3, false)
