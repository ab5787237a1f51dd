// kern_f64_r4_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r4_abl, double, 4)
