// kern_f32_r3_ws.cu -- warp-specialized in-plane sweep instantiations
// (inplane_ws.cuh) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_WS(register_f32_r3_ws, float, 3, false)
