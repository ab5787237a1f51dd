// kern_f32_r3_dg.cu -- Div / Grad application stencils (divgrad.cuh) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f32_r3_dg, float, 3)
