// kern_f64_r3_g.cu -- application-stencil sweep kernels (second, centre-only
// input grid; Table V) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r3_g, double, 3, true)
