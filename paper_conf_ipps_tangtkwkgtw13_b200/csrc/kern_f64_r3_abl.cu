// kern_f64_r3_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f64_r3_abl, double, 3)
