// kern_f32_r4_dg.cu -- Div / Grad application stencils (divgrad.cuh) for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f32_r4_dg, float, 4)
