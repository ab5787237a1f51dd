// kern_f32_r4_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f32_r4_ps, float, 4)
