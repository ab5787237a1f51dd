// kern_f32_r2.cu -- sweep-kernel instantiations for float, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r2, float, 2, false)
