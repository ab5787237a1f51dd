// kern_f64_r2_ps.cu -- fused peer-store halo-exchange sweep kernels (p2p slab plans) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_PS(register_f64_r2_ps, double, 2)
