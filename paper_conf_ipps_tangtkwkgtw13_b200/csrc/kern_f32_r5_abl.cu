// kern_f32_r5_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r5_abl, float, 5)
