// kern_f32_r2_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r2_ws, float, 2, false)
