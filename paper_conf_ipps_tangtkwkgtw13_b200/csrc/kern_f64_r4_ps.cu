// kern_f64_r4_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f64_r4_ps, double, 4)
