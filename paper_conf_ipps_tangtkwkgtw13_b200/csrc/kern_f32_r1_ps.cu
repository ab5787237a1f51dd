// kern_f32_r1_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f32_r1_ps, float, 1)
