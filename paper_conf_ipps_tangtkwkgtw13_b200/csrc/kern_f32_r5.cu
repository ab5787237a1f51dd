// kern_f32_r5.cu -- sweep-kernel instantiations for float, r = 5 (Table IV order 10).
#include "kern_inst.cuh"
STENCIL_REGISTER(register_f32_r5, float, 5, false)
