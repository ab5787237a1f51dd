// kern_f64_r4.cu -- sweep-kernel instantiations for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r4, double, 4, false)
