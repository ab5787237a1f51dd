// kern_f32_r4.cu -- sweep-kernel instantiations for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r4, float, 4, false)
