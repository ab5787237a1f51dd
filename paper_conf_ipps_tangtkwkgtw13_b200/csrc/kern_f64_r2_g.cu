// kern_f64_r2_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r2_g, double, 2, true)
