// kern_f64_r6_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for double, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f64_r6_ps, double, 6)
