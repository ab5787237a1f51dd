// kern_f64_r6_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for double, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r6_g, double, 6, true)
