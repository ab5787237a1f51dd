// kern_f64_r5.cu -- sweep-kernel instantiations for double, r = 5 (Table IV order 10).
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r5, double, 5, false)
