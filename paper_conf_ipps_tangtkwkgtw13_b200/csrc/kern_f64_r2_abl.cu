// kern_f64_r2_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r2_abl, double, 2)
