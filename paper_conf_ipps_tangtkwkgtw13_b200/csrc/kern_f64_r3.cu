// kern_f64_r3.cu -- sweep-kernel instantiations for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r3, double, 3, false)
