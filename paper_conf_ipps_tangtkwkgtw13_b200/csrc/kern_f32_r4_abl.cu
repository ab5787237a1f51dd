// kern_f32_r4_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r4_abl, float, 4)
