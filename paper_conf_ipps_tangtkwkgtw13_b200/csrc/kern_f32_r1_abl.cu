// kern_f32_r1_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r1_abl, float, 1)
