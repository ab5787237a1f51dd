// kern_f64_r6.cu -- sweep-kernel instantiations for double, r = 6 (Table IV order 12).
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f64_r6, double, 6, false)
