// kern_f32_r6_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for float, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r6_g, float, 6, true)
