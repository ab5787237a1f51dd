// kern_f64_r2.cu -- sweep-kernel instantiations for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r2, double, 2, false)
