// kern_f32_r1_dg.cu -- Div / Grad application stencils (divgrad.cuh) for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f32_r1_dg, float, 1)
