// kern_f32_r4_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r4_ws, float, 4, false)
