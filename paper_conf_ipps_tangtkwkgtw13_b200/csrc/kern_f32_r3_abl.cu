// kern_f32_r3_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r3_abl, float, 3)
