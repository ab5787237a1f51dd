// kern_f64_r4_dg.cu -- Div / Grad application stencils (divgrad.cuh) for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f64_r4_dg, double, 4)
