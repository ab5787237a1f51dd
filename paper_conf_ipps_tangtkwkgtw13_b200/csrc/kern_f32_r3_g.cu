// kern_f32_r3_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r3_g, float, 3, true)
