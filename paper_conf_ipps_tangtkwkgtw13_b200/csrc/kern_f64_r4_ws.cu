// kern_f64_r4_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f64_r4_ws, double, 4, false)
