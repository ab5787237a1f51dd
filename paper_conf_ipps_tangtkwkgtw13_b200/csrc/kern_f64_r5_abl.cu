// kern_f64_r5_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r5_abl, double, 5)
