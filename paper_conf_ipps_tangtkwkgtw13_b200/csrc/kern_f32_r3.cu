// kern_f32_r3.cu -- sweep-kernel instantiations for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r3, float, 3, false)
