// kern_f32_r2_dg.cu -- Div / Grad application stencils (divgrad.cuh) for float, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f32_r2_dg, float, 2)
