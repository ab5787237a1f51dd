// kern_f32_r1_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r1_ws, float, 1, false)
