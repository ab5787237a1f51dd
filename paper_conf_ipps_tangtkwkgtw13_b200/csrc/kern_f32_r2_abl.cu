// kern_f32_r2_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r2_abl, float, 2)
