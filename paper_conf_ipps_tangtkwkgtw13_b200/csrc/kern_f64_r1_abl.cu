// kern_f64_r1_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r1_abl, double, 1)
