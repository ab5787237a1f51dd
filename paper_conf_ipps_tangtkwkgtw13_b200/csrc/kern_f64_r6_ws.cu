// kern_f64_r6_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r6_ws, double, 6, false)
