// kern_f64_r5_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for double, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r5_g, double, 5, true)
