// kern_f32_r6_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r6_ws, float, 6, false)
