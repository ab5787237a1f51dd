// kern_f32_r6_abl.cu -- ablation kernels (ablation.cuh, forward.cuh with
// register rows) for float, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_ABL(register_f32_r6_abl, float, 6)
