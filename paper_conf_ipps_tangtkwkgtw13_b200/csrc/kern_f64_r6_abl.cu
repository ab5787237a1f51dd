// kern_f64_r6_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r6_abl, double, 6)
