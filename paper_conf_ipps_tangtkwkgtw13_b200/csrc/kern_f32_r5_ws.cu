// kern_f32_r5_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r5_ws, float, 5, false)
