// kern_f64_r3_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f64_r3_ps, double, 3)
