// kern_f32_r1.cu -- sweep-kernel instantiations for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r1, float, 1, false)
