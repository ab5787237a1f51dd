// kern_f64_r1.cu -- sweep-kernel instantiations for double, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r1, double, 1, false)
