// kern_f32_r6.cu -- sweep-kernel instantiations for float, r = 6 (Table IV order 12).
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r6, float, 6, false)
