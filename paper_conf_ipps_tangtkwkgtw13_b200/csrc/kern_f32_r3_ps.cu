// kern_f32_r3_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f32_r3_ps, float, 3)
